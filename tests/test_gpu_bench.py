"""Bit-exactness at the bench's own configuration (BASELINE configs[4], C5: the ResNet-50
trunk at batch 256 on one GPU), byte for byte against the CPU oracle:

* the chained trunk exactly as bench.py builds and launches it (same descriptors, weights,
  plans -- including the 4-bit BN = 256 tiles of the im2col and CTA-pair kernels and their
  128-byte int4 output staging), images 0 and 255 through the oracle's chain of all 53
  layers, every layer's output compared;
* every trunk layer again with freshly drawn inputs (images 0, 128, 255), so a layer is
  also checked on inputs its predecessor did not produce;
* the chained trunk at batch 2 (small plans).
"""
import numpy as np
import pytest

import oracle
import workloads as W

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA GPU", allow_module_level=True)

import bench  # noqa: E402
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402

DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module", params=[(4, False), (8, False), (4, True), (8, True)],
                ids=["a4w4", "a8w8", "a4w4-tuned", "a8w8-tuned"])
def trunk256(request):
    """The bench trunk with the default kernel rule, and with the committed tile-search table
    (plans/, what bench.py loads by default)."""
    import os
    from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning
    bits, tuned = request.param
    qc.qconv_plan_clear()
    if tuned:
        path = os.path.join(os.path.dirname(bench.__file__), "plans", f"resnet50_trunk_a{bits}_b256.json")
        if not os.path.exists(path):
            pytest.skip("no tile-search table committed")
        assert tuning.load_plans(path) > 40
    t = bench.Trunk(bits, 256, DEV)
    t.step()
    torch.cuda.synchronize()
    yield t
    qc.qconv_plan_clear()
    del t
    torch.cuda.empty_cache()


def test_trunk256_plans_cover_the_wide_tiles(trunk256):
    plans = [(L["plan"]["kernel_name"], L["plan"]["bn"]) for L in trunk256.layers]
    assert ("pair", 256) in plans
    assert {"halo_t", "channel"} <= {k for k, _ in plans}


def test_trunk256_chain_vs_oracle(trunk256):
    res = bench.verify_trunk(trunk256, [0, 255])
    assert res["bit_exact"], res["mismatch"]


def test_trunk256_every_layer_fresh_inputs(trunk256):
    bits = trunk256.bits
    ot = bench.OracleTrunk(bits)
    for j, L in enumerate(trunk256.layers):
        if j == 0:
            continue                                 # the stem: covered by the chain test
        cs = L["shape"]
        x = W.device_post_relu_codes(tuple(L["x"].shape[:3]) + (cs.c,), bits, 9000 + j, DEV)
        y = qc.qconv2d_forward(L["desc"], x, L["w"], L["bias"], L["m"], L["n"])
        torch.cuda.synchronize()
        for img in (0, 128, 255):
            ref = ot._run_layer(j, x[img:img + 1].cpu().numpy())
            got = y[img:img + 1].cpu().numpy()
            if not np.array_equal(got, ref):
                raise AssertionError(f"{L['name']} ({L['plan']['kernel_name']} bn={L['plan']['bn']}) "
                                     f"img {img}: {(got != ref).sum()} bytes differ")


@pytest.mark.parametrize("bits", [4, 8])
def test_trunk_batch2_chain_vs_oracle(bits):
    t = bench.Trunk(bits, 2, DEV)
    t.step()
    torch.cuda.synchronize()
    res = bench.verify_trunk(t, [0, 1])
    assert res["bit_exact"], res["mismatch"]
