"""GPU parity at the bench / BASELINE full sizes on sampled outputs (the launch configuration
bench.py times), plus cutcp at the config-3 water box."""
import pytest
import torch

pytestmark = pytest.mark.gpu

from tests.gpu_helpers import be_case, host  # noqa: E402


@pytest.fixture(scope="module")
def tk():
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker
    assert torch.cuda.is_available()
    return tacker


@pytest.mark.parametrize("kind", ["BE_CUTCP", "BE_MRIQ_Q", "BE_STENCIL", "BE_LBM", "BE_MRIFHD_FH", "BE_CP", "BE_FFT", "BE_TPACF"])
def test_full_size_original_and_fused(tk, kind):
    import synth
    from tests.gpu_helpers import dev, t
    c = be_case(getattr(tk, kind), seed=11, size="large")
    c["reset"]()
    tk.tacker_launch_original(None, c["desc"])
    orig = [host(o).copy() for o in c["outs"]]
    c["check"](orig)
    A, B = synth.lc_gemm_inputs(512, 256, 256, seed=0)
    D = torch.zeros(512, 256, device=dev())
    for ws in ((20 if kind != "BE_CUTCP" else 24), 8):   # default and register-rich class
        f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], ws)
        c["reset"]()
        f.launch()
        for a, o in zip(orig, c["outs"]):
            assert a.tobytes() == host(o).tobytes()
