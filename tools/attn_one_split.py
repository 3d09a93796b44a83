"""One KV-split attention launch (for ncu), the step's configuration: python tools/attn_one_split.py L H D"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

L, H, D = (int(a) for a in sys.argv[1:4])
qkv = torch.randn(L, 3 * H * D, device="cuda").to(torch.bfloat16)
o = torch.empty(L, H * D, dtype=torch.bfloat16, device="cuda")
cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
ws = torch.empty(32 << 20, dtype=torch.float32, device="cuda")
ld = 3 * H * D
for _ in range(2):
    tsv.op_attention_split(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, cnt, ws, nsplit=0, ldq=ld, ldk=ld, ldv=ld)
torch.cuda.synchronize()
