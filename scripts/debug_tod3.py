import numpy as np
import torch
from paper_conf_sc_demeurekktbb23_b200 import binding, synth
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload

w = synth.make_workload("c1", n_det=1, n_samp=256, nnz=1, nside=4096)
w.det_scale = np.ones(1)
tod = 2.0 ** np.arange(256)[None, :] * 0 + np.arange(256)[None, :] * 1.0 + 1000
w.det_data = np.ascontiguousarray(tod)
dw = DeviceWorkload.upload(w, "cuda")
pix = torch.full((1, w.n_samp), -7, dtype=torch.int64, device="cuda")
dw.pointing_to_map(pixels_out=pix)
torch.cuda.synchronize()
pg = pix.cpu().numpy()[0]
z = dw.zmap.cpu().numpy().reshape(-1)
print("intervals", w.intervals[:3], "path", binding.last_fused_path())
runs = []
s = 0
while s < 256:
    e = s
    while e + 1 < 256 and pg[e + 1] == pg[s]:
        e += 1
    runs.append((s, e, pg[s]))
    s = e + 1
for s, e, p in runs[:40]:
    exp = tod[0, s:e + 1].sum()
    print(f"samples {s:3d}-{e:3d} pix {p} got {z[p]:.0f} exp {exp:.0f} diff {z[p]-exp:.0f}")
