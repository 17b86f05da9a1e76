"""Host-buffer TM with frame streaming (the paper's per-frame runtime operation,
5.1.3.4 P:91): ncc_match_host with more frames than one chunk copies chunk c + 1 on the plan's
copy stream while chunk c is matched.  Peaks and surfaces must equal the device path bit for
bit (tensor-core, CUDA-core and tiny plans), over repeated calls that reuse the two slots."""
import numpy as np
import pytest
import torch

import synth
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


@pytest.mark.parametrize("shape,kw,chunk", [((1024, 1024, 128, 128), {}, "2"),
                                            ((1024, 1024, 128, 128), {}, None),
                                            ((300, 280, 24, 20), {"cuda_cores": True}, "2"),
                                            ((64, 64, 16, 16), {}, "3")])
def test_streamed_host_batch_equals_device_path(shape, kw, chunk, monkeypatch):
    if chunk:
        monkeypatch.setenv("NCC_TM_CHUNK", chunk)
    H, W, h, w = shape
    F = 5
    imgs = np.stack([synth.uniform_image(H, W, 9300 + k) for k in range(F)])
    T, u0, v0 = synth.planted_template(imgs[3], h, w, 9400)
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, batch=F, write_surface=True, **kw) as plan:
        pk_d, sc_d = plan.match(torch.from_numpy(imgs).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
        pk_d, sc_d = pk_d.cpu().numpy(), sc_d.cpu().numpy()
        hi = torch.from_numpy(imgs).pin_memory()
        ht = torch.from_numpy(T).pin_memory()
        hp = torch.full((F, 4), -1, dtype=torch.int32).pin_memory()
        hs = torch.zeros((F, plan.band_rows, plan.info.V), dtype=torch.float32).pin_memory()
        for _ in range(3):
            plan.match_host(hi, ht, hp, h_scores=hs)
        torch.cuda.synchronize()
    np.testing.assert_array_equal(hp.numpy(), pk_d)
    np.testing.assert_array_equal(hs.numpy(), sc_d)
    d = decode_peaks(hp)
    assert (int(d["u"][3]), int(d["v"][3])) == (u0, v0)
