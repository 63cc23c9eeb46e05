"""f3: the Fig 1 memory-copy microbenchmark kernels copy exactly."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import synth
from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C
from test_gpu_parity import assert_exact, dev, host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()
    C.load()


def test_memcopy_variants_exact():
    C.cudanp_dp_set_pending_launch_limit(1 << 17)
    C.cudanp_dp_error_count(reset=True)
    x = synth.gen(1, "f32_signed", 0, 1 << 20)
    xd = dev(x)
    for variant, ms in ((0, [1]), (1, [1]), (2, [1, 64, 4096, 1 << 16])):
        for m in ms:
            out = torch.full_like(xd, float("nan"))
            C.cudanp_dp_memcopy(xd, out, m=m, variant=variant)
            assert_exact(host(out), x, f"variant={variant} m={m}")
    assert C.cudanp_dp_error_count(reset=True) == 0
    with pytest.raises(C.CudanpError):
        C.cudanp_dp_memcopy(xd, m=3, variant=2)  # m must divide the element count
