"""One launch of each HBM-bound kernel at the bench's per-microbatch token
count (T = mbs 32 x s 1024 = 32768, h = 1600, V = 50304), for an
`ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum`
capture (DRAM evidence for the fused elementwise kernels).
Each kernel sees fresh (cold) inputs larger than L2."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

T, h, V, s = int(os.environ.get("ELEM_T", "32768")), 1600, 50304, 1024
mk = lambda *sh: torch.randn(*sh, device="cuda").to(torch.bfloat16)  # noqa: E731
x, dy, dres, g, b = mk(T, h), mk(T, h), mk(T, h), mk(h), mk(h)
y, dx = torch.empty_like(x), torch.empty_like(x)
mu, rs = torch.empty(T, device="cuda"), torch.empty(T, device="cuda")
dg, db = torch.zeros(h, device="cuda"), torch.zeros(h, device="cuda")
kt.layernorm_fwd(BF16, x, g, b, y, mu, rs, T, h)
kt.layernorm_bwd(BF16, dy, x, g, mu, rs, dres, dx, dg, db, T, h)
for n in (h, 3 * h, 4 * h):
    X = mk(T, n)
    kt.colsum(BF16, X, n, T, n, torch.zeros(n, device="cuda"))
    del X
rows = T // 4  # CE on a quarter of the logits (the full [T, V] bf16 is 3.3 GB)
z = mk(rows, V)
tok = torch.randint(0, V, (rows // s, s + 1), device="cuda", dtype=torch.int32)
kt.cross_entropy(BF16, z, tok, torch.empty(rows, device="cuda"), rows, V, s, 1.0 / rows)
del z
tokT = torch.randint(0, V, (T // s, s + 1), device="cuda", dtype=torch.int32)
wte, wpe = mk(V, h), mk(s, h)
kt.embed_fwd(BF16, tokT, wte, wpe, y, T // s, s, h)
kt.embed_bwd(BF16, tokT, dy, torch.zeros(V, h, device="cuda"), torch.zeros(s, h, device="cuda"), T // s, s, h, V)
# flash backward pre / post passes (dsum + dQ zeroing, dQ cast) come with one attention call
qkv, o, do, dq = mk(T, 3 * h), mk(T, h), mk(T, h), mk(T, 3 * h)
kt.attention(BF16, T // s, s, 25, 64, qkv, o, do, dq)
torch.cuda.synchronize()
print("done")
