"""The round-1 task variant "ozaki" (Ozaki scheme I: INT8 slices of A and B,
S(S+1)/2 slice products) is retired.  Its dropped slice products bound the error
only by ~(S-1) 2^-7S K max|a_i| max|b_j| (2^-42 at S = 6), which cannot certify
the componentwise 1e-12 bar against D = |A||B| (R19, R21); the FP64
INT8 path is Ozaki scheme II with its certificate (test_gpu_ozaki2.py).  A
descriptor that still names the variant gets PDL_EUNSUPPORTED at pdl_run, for
FP64 (DGEMM_VARIANT) and FP32 (SGEMM_VARIANT) tasks alike."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    for k in ("PDL_DRY_RUN", "PDL_DGEMM_VARIANT", "PDL_SGEMM_VARIANT"):
        monkeypatch.delenv(k, raising=False)
    pdl.unload()
    yield
    pdl.unload()


@pytest.mark.parametrize("dt,prop", [(torch.float64, "DGEMM_VARIANT"), (torch.float32, "SGEMM_VARIANT")])
def test_ozaki_scheme_one_is_retired(dt, prop):
    pdl.load(pdl.descriptor_xml(1, props={prop: "ozaki"}))
    A = torch.rand((64, 64), dtype=dt, device="cuda")
    C = torch.empty((64, 64), dtype=dt, device="cuda")
    pdl.task_matmul(A, A, C)
    with pytest.raises(pdl.PDLError) as e:
        pdl.run()
    assert e.value.code == pdl.PDL_EUNSUPPORTED
    assert "retired" in str(e.value)
    # the library stays usable: the default variant runs
    pdl.unload()
    pdl.load(pdl.descriptor_xml(1))
    pdl.task_matmul(A, A, C)
    pdl.run()
    tol = 1e-12 if dt == torch.float64 else 1e-5
    ref = (A.double() @ A.double())
    assert ((C.double() - ref).abs() <= tol * (A.double().abs() @ A.double().abs())).all()
