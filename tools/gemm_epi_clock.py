"""Run one fc1-shape GEMM epilogue variant back to back for ~3 s while
sampling the SM clock (nvidia-smi): separates power-capped clock drops from
per-tile epilogue cost.  Research tool."""
import os
import subprocess
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MOBIUS_KT_NOSYNC", "1")
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

T, h = 32768, 1600
M, N, K = T, 4 * h, h
mk = lambda *s: (torch.randn(*s, device="cuda") * 0.1).to(torch.bfloat16)  # noqa: E731
A, B, bias = mk(M, K), mk(K, N), mk(N)
C, X = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16), torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
for epi in (1, 2, 1, 2):
    fn = lambda: kt.gemm(BF16, M, N, K, A, K, False, B, N, True, C, N, epi=epi, bias=bias,  # noqa: E731
                         AUX=X if epi == 2 else None, ldx=N)
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    clocks, stop = [], [False]

    def sample():
        while not stop[0]:
            o = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm,power.draw", "--format=csv,noheader,nounits"],
                               capture_output=True, text=True).stdout.strip()
            clocks.append(o)
            time.sleep(0.1)
    th = threading.Thread(target=sample)
    th.start()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 6000
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    stop[0] = True
    th.join()
    us = a.elapsed_time(b) / n * 1e3
    mid = clocks[len(clocks) // 4: 3 * len(clocks) // 4] or clocks
    print(f"epi {epi}: {us:7.1f} us {2.0 * M * N * K / us / 1e6:6.0f} TF/s  clocks/power {mid[:3]} .. {mid[-2:]}")
