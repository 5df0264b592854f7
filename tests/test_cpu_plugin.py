"""The paper's CPU decoder variant (scripts/cpu_plugin.c, a comparison point
only: SURVEY.md §8f f4) decodes the product's streams to the
same bits as the CPU oracle (no GPU needed)."""
import sys
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT / "scripts"))


def test_cpu_plugin_matches_oracle(orc):
    import cpu_plugin
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    L = cpu_plugin.load(native=False)
    for x, loc in ((gen_cosmo(1001, n=64), False), (gen_cosmo(3002, "dense", n=64), False),
                   (gen_cosmo(3001, "sparse", n=64), True), (np.zeros((4, 8, 16, 16), np.int16), False)):
        b = spp.spp_encode_cosmo(x, localize=loc)
        got = cpu_plugin.cosmo_decode(L, b, x.shape)
        assert np.array_equal(got.view(np.uint16), orc.cosmo_direct(x, 1, "f16").view(np.uint16))
    y = gen_deepcam(2001, H=24)
    y[3, 5, 7] = np.nan                                    # a RAW line
    mean, rstd = deepcam_stats(np.nan_to_num(y))
    for d in (spp.spp_encode_deepcam(y), spp.spp_encode_deepcam(y, err_budget=4),
              spp.spp_encode_deepcam(y, err_budget=4, raw16=True)):
        got = cpu_plugin.deepcam_decode(L, d, y.shape, mean, rstd)
        want = orc.deepcam_decode(d, y.shape, mean, rstd, "f16")
        nan = np.isnan(want)
        assert np.array_equal(np.isnan(got), nan)
        assert np.array_equal(got[~nan].view(np.uint16), want[~nan].view(np.uint16))
