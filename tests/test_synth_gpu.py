"""The on-device timestream generator (bench / test input, include/toast_b200_synth.h) is
bit-identical to the host generator synth.tod_rows on subsets of every config's detectors."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from paper_conf_sc_demeurekktbb23_b200 import binding, synth  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name,obs", [("c2", 0), ("c4", 0), ("c5", 7)])
def test_device_tod_equals_host_generator(name, obs):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    w = synth.make_workload(name, n_samp=50_000, obs=obs, with_tod=False, det_range=(3, 41))
    out = torch.empty((w.n_det, w.n_samp), dtype=torch.float64, device="cuda")
    binding.synth_tod(out, torch.from_numpy(w.sigma).cuda(), torch.from_numpy(w.det_ids).cuda(), w.seed)
    host = synth.tod_rows(w.seed, w.sigma, w.det_ids, w.n_samp)
    np.testing.assert_array_equal(out.cpu().numpy(), host)
