"""The tuning cache (STENCIL_TUNE_CACHE, stencil.h stencil_tune) and the sustained-clock report."""
import os

import pytest

import stencil_inputs as si

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def test_cache_written_and_used(S, tmp_path, monkeypatch):
    import torch
    path = tmp_path / "cache.txt"
    monkeypatch.setenv("STENCIL_TUNE_CACHE", str(path))
    r, n = 2, 96
    c = si.coeffs_as("heat", r, "f32")
    with S.Plan(n, n, n, r, c, "f32") as p:
        s0, s1 = p.alloc(), p.alloc()
        p.fill_counter(s0, 1)
        s1.copy_(s0)
        rep = p.tune(kernel="inplane_ws", beta=5, iters_per_rep=2, reps=1, scratch=(s0, s1))
        tuned = p.config
        assert rep["best_measured_gpts"] > 0 and rep["best_burst_gpts"] > 0
    lines = path.read_text().split("\n")
    assert lines[0].startswith("stencil-tune-v1 0 2 96 96 96 0 ")
    with S.Plan(n, n, n, r, c, "f32") as q:          # a new plan of the same problem starts from the cache
        assert q.config == tuned
    with S.Plan(n, n, n + 1, r, c, "f32") as q:      # another problem does not
        assert q.config["kernel"] in ("inplane", "inplane_ws")
    torch.cuda.synchronize()


def test_cache_ignores_invalid_lines(S, tmp_path, monkeypatch):
    path = tmp_path / "cache.txt"
    path.write_text("garbage line\nstencil-tune-v1 0 1 40 40 40 0 148 2 16 4 4 2 3 1 2 0 1.0\n"
                    "stencil-tune-v1 0 1 40 40 40 0 148 2 20 4 4 2 3 1 2 0 99.0\n")   # tx=20 invalid
    monkeypatch.setenv("STENCIL_TUNE_CACHE", str(path))
    import torch
    sm = torch.cuda.get_device_properties(0).multi_processor_count
    if sm != 148:
        pytest.skip("cache lines are keyed by a 148-SM device")
    with S.Plan(40, 40, 40, 1, si.coeffs_as("heat", 1, "f32"), "f32") as p:
        cfg = p.config
        assert (cfg["kernel"], cfg["tx"], cfg["ty"], cfg["ry"], cfg["zbox"]) == ("inplane_ws", 16, 4, 2, 2)
