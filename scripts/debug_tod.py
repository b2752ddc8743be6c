"""GPU debug: the fused map with a ramp TOD against np.add.at over the kernel's own pixels."""
import numpy as np
import torch
from paper_conf_sc_demeurekktbb23_b200 import binding, synth
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload

for n_det in (4, 40):
    w = synth.make_workload("c1", n_det=n_det, n_samp=4096, nnz=1)
    w.det_scale = np.ones(n_det)
    for kind in ("ones", "ramp"):
        tod = np.ones((n_det, w.n_samp)) if kind == "ones" else (np.arange(w.n_samp)[None, :] + 1000.0 * np.arange(n_det)[:, None])
        w.det_data = np.ascontiguousarray(tod)
        dw = DeviceWorkload.upload(w, "cuda")
        pix = torch.full((n_det, w.n_samp), -7, dtype=torch.int64, device="cuda")
        dw.pointing_to_map(pixels_out=pix)
        torch.cuda.synchronize()
        pg = pix.cpu().numpy()
        exp = np.zeros(w.npix)
        np.add.at(exp, pg[pg >= 0], tod[pg >= 0])
        got = dw.zmap.cpu().numpy().reshape(-1)
        bad = np.nonzero(np.abs(got - exp) > 1e-9 * (1 + np.abs(exp)))[0]
        print(n_det, kind, "path", binding.last_fused_path(), "bad", len(bad), "of", int((exp != 0).sum()),
              "sum got", got.sum(), "exp", exp.sum())
        if len(bad):
            print("  first bad pixels", bad[:5], got[bad[:5]], exp[bad[:5]])
