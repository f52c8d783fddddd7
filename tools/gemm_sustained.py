"""Per-shape GEMM A/B, ours vs cuBLAS (torch.matmul, bf16 out, no fused
epilogue), each run back to back for ~1.5 s so the GPU sits at its power cap
as it does inside a training step (the burst A/B in gemm_vs_cublas.py runs
at higher clocks).  Prints us / TF/s and the median SM clock of each run.
Kernel-level tool, not part of the bench contract."""
import os
import subprocess
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MOBIUS_KT_NOSYNC", "1")
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402
from tools.gemm_prof import SHAPES  # noqa: E402


def sustained(fn, seconds=1.5):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fn()
    b.record()
    torch.cuda.synchronize()
    n = max(10, int(seconds / (a.elapsed_time(b) * 1e-3)))
    clocks, stop = [], [False]

    def sample():
        while not stop[0]:
            o = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv,noheader,nounits"],
                               capture_output=True, text=True).stdout.strip()
            if o:
                clocks.append(int(o.split()[0]))
            time.sleep(0.05)
    th = threading.Thread(target=sample)
    th.start()
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    stop[0] = True
    th.join()
    cl = sorted(clocks[len(clocks) // 3:]) or [0]
    return a.elapsed_time(b) / n * 1e3, cl[len(cl) // 2]


def mk(*s):
    return (torch.randn(*s, device="cuda") * 0.1).to(torch.bfloat16)


tot_o = tot_c = 0.0
for name, M, N, K, amn, bmn, epi, cf in SHAPES:
    A = mk(K, M) if amn else mk(M, K)
    B = mk(K, N) if bmn else mk(N, K)
    C = torch.zeros(M, N, device="cuda", dtype=torch.float32 if cf else torch.bfloat16)
    bias, R, AUX = mk(N), mk(M, N), mk(M, N)
    ours, co = sustained(lambda: kt.gemm(BF16, M, N, K, A, M if amn else K, amn, B, N if bmn else K, bmn, C, N,
                                         c_f32=bool(cf), epi=epi, bias=bias if epi in (1, 2, 3) else None,
                                         R=R if epi in (3, 4) else None, ldr=N, AUX=AUX if epi == 2 else None,
                                         ldx=N, accumulate=(epi == 5)))
    Am = A.t() if amn else A
    Bm = B if bmn else B.t()
    Cb = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    cub, cc = (1.0, 0) if os.environ.get("OURS_ONLY") else sustained(lambda: torch.matmul(Am, Bm, out=Cb))
    fl = 2.0 * M * N * K
    tot_o += ours
    tot_c += cub
    print(f"{name:18s} {M:6d}x{N:6d}x{K:6d}  ours {ours:7.1f} us {fl / ours / 1e6:6.0f} TF/s @{co} MHz   "
          f"cublas {cub:7.1f} us {fl / cub / 1e6:6.0f} TF/s @{cc} MHz   ratio {cub / ours:.2f}", flush=True)
print(f"total ours {tot_o:.0f} us, cublas {tot_c:.0f} us")
