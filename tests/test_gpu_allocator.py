"""Caller-supplied device memory (cd_options.alloc / free / alloc_ctx; PyTorch
supplies the memory): every device buffer of a call comes from PyTorch's caching allocator, the
results are identical to the pool-backed path, and everything is returned."""
import ctypes as C

import numpy as np
import pytest

from tools import popgen

pytestmark = pytest.mark.gpu

cds = pytest.importorskip("paper_conf_ipps_hellwigcmbw23_b200")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@pytest.mark.parametrize("mode,dt", [("grid", 1.0), ("hybrid", 9.0), ("legacy", 1.0)])
def test_torch_allocator_same_result(mode, dt):
    import torch
    pop = popgen.random_population(20000, 91, "catalog", 4000)
    t1 = 300.0 * dt
    ref = cds.screen(pop, 0.0, t1, dt, 5.0, mode=mode)
    torch.cuda.synchronize()
    before = torch.cuda.memory_allocated()
    stream = torch.cuda.current_stream().cuda_stream
    al = cds.TorchAllocator(torch.cuda.current_device(), stream)
    got = cds.screen(pop, 0.0, t1, dt, 5.0, mode=mode, allocator=al, stream=stream)
    torch.cuda.synchronize()
    assert len(ref) > 10
    assert np.array_equal(got, ref)
    assert al.calls > 5 and al.live == 0
    assert torch.cuda.memory_allocated() == before


def test_torch_allocator_device_results_and_candidates():
    import torch
    pop = popgen.random_population(8000, 92, "catalog", 1000)
    stream = torch.cuda.current_stream().cuda_stream
    al = cds.TorchAllocator(torch.cuda.current_device(), stream)
    E = cds._Elements(pop)
    opt = cds.make_options(outputs_on_device=True, stream=stream, allocator=al)
    out = cds.cd_conjunctions()
    cds._check(cds.cd_screen_ex(E.s, E.n, 0.0, 200.0, 1.0, 10.0, cds.CD_GRID, opt, out))
    n = int(out.count)
    assert n > 0 and al.live == 1          # the device result is the caller's block
    cds.cd_conjunctions_free(out)
    torch.cuda.synchronize()
    assert al.live == 0
    K1 = cds.candidates(pop, 0.0, 200.0, 1.0, 10.0)
    K2 = cds.candidates(pop, 0.0, 200.0, 1.0, 10.0, allocator="torch")
    assert np.array_equal(K1, K2)


def test_allocator_errors():
    pop = popgen.random_population(2000, 93)
    E = cds._Elements(pop)
    opt = cds.make_options()
    opt.alloc = cds.ALLOC_FN(lambda n, ctx: None)   # alloc without free
    out = cds.cd_conjunctions()
    assert cds.cd_screen_ex(E.s, E.n, 0.0, 10.0, 1.0, 5.0, cds.CD_GRID, opt, out) == cds.CD_EINVAL

    class Failing(cds.TorchAllocator):
        pass
    import torch
    al = Failing(torch.cuda.current_device(), torch.cuda.current_stream().cuda_stream)
    n_ok = [0]
    base_alloc = al.c_alloc

    def flaky(nbytes, ctx):
        n_ok[0] += 1
        return base_alloc(nbytes, ctx) if n_ok[0] < 4 else None
    al.c_alloc = cds.ALLOC_FN(flaky)
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 10.0, 1.0, 5.0, allocator=al, stream=al.stream)
    assert ei.value.status in (cds.CD_ENOMEM, cds.CD_ECUDA)
    torch.cuda.synchronize()
    assert al.live == 0
