"""One attention launch (for ncu): python tools/attn_one.py L H D impl"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

L, H, D, impl = (int(a) for a in sys.argv[1:5])
qkv = torch.randn(L, 3 * H * D, device="cuda").to(torch.bfloat16)
o = torch.empty(L, H * D, dtype=torch.bfloat16, device="cuda")
ld = 3 * H * D
for _ in range(2):
    tsv.op_attention(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, ldq=ld, ldk=ld, ldv=ld, impl=impl)
torch.cuda.synchronize()
