"""Small steps covering every kernel path, for compute-sanitizer (tools/gpurun_sanitize.sh): tiny FLUX
with single blocks, tiny SD3 (D = 64 attention, CFG pair), SP = 2 / 4 on virtual ranks with the
fused and the exchange transports, a reshard, a batched step."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_luhtlwm0c26_b200 as tsv  # noqa: E402

for model in ("tiny2", "tiny_sd3"):
    for fused in (True, False):
        eng = tsv.Engine(model, devices=[0] * 4)
        eng.set_transport(fused)
        g1, g2, g4 = eng.group_create([0]), eng.group_create([1, 0]), eng.group_create([0, 1, 2, 3])
        r = eng.request_create(208, 240, num_steps=4, seed=7)
        for s, g in enumerate([g1, g2, g4]):
            eng.request_step(r, s, g)
        b = [eng.request_create(208, 240, num_steps=2, seed=8 + i) for i in range(2)]
        eng.event_wait(eng.request_step_batch(b, g2))
        print(model, fused, float(abs(eng.read_latent(r)).max()), flush=True)
        eng.close()

# the attention's KV split with a tail (whole items first, the last items in key ranges: FLUX / SD3
# 1024^2 at SP = 2 shapes) and the uniform split, kernel-level
import torch  # noqa: E402

for L, H, D in ((4608, 12, 128), (4429, 12, 64)):
    for nsplit in (0, 3):
        qkv = torch.randn(L, 3 * H * D, device="cuda").to(torch.bfloat16)
        o = torch.zeros(L, H * D, dtype=torch.bfloat16, device="cuda")
        cnt = torch.zeros(4096, dtype=torch.int32, device="cuda")
        ws = torch.empty(32 << 20, dtype=torch.float32, device="cuda")
        ld = 3 * H * D
        tsv.op_attention_split(qkv, qkv[:, H * D:], qkv[:, 2 * H * D:], o, L, H, D, cnt, ws, nsplit=nsplit, ldq=ld,
                               ldk=ld, ldv=ld)
        torch.cuda.synchronize()
        print("attention split", L, H, D, nsplit, float(o.float().abs().max()), int(torch.count_nonzero(cnt)), flush=True)
