"""CPU-side checks of the C-ABI library (no compute calls): it loads, exports every symbol
include/cdscreen.h declares, its structs have the declared layout, and without a GPU every
compute entry point fails loudly (no CPU fallback)."""
import ctypes as C
import re
import subprocess
from pathlib import Path

import numpy as np
import pytest

ROOT = Path(__file__).resolve().parent.parent
HEADER = ROOT / "include" / "cdscreen.h"


@pytest.fixture(scope="module")
def cds():
    from paper_conf_ipps_hellwigcmbw23_b200 import _build
    _build.build()
    import paper_conf_ipps_hellwigcmbw23_b200 as m
    m.lib()
    return m


def declared_functions():
    txt = HEADER.read_text()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:[A-Za-z_][\w\s\*]*?)\b(cd_\w+)\s*\(", txt, flags=re.M)))


def test_exports_every_declared_symbol(cds):
    names = declared_functions()
    assert "cd_screen" in names and "cd_propagate" in names and len(names) >= 11
    out = subprocess.run(["nm", "-D", "--defined-only", str(cds.LIB_PATH)], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\b(cd_\w+)\b", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    L = cds.lib()
    for n in names:
        assert hasattr(L, n)
    assert set(names) == set(cds.ABI_SYMBOLS)


def test_version_status_options(cds):
    assert cds.cd_abi_version() == cds.ABI_VERSION
    assert cds.status_str(cds.CD_EINVAL) == "CD_EINVAL"
    assert cds.status_str(cds.CD_ENODEV) == "CD_ENODEV"
    o = cds.cd_options()
    cds.cd_options_init(o)
    assert o.v_margin == 7.8 and o.n_ranks == 1 and o.cell_factor == 0.0 and o.device == -1


def test_struct_layouts(cds):
    assert C.sizeof(cds.cd_conjunction) == 32 and cds.CONJ_DTYPE.itemsize == 32
    assert C.sizeof(cds.cd_candidate) == 12 and cds.CAND_DTYPE.itemsize == 12
    assert C.sizeof(cds.cd_elements) == 48


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.mark.skipif(_has_gpu(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback(cds):
    pop = {k: np.ones(4) * v for k, v in zip(cds.FIELDS, (7000.0, 0.001, 1, 1, 1, 1))}
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 10.0, 1.0, 2.0)
    assert ei.value.status == cds.CD_ENODEV
    with pytest.raises(cds.CdError) as ei:
        cds.propagate(pop, [0.0])
    assert ei.value.status == cds.CD_ENODEV


def test_option_validation_before_device(cds):
    """Invalid options are CD_EINVAL on any machine (validated before a device is touched)."""
    pop = {k: np.ones(4) * v for k, v in zip(cds.FIELDS, (7000.0, 0.001, 1, 1, 1, 1))}
    for kw in (dict(kepler_points=5), dict(kepler_points=-4), dict(cell_factor=0.5),
               dict(rank=2, n_ranks=2)):
        with pytest.raises(cds.CdError) as ei:
            cds.screen(pop, 0.0, 10.0, 1.0, 2.0, **kw)
        assert ei.value.status == cds.CD_EINVAL, kw
    assert cds.cd_release_caches(-1) == cds.CD_OK or _has_gpu()


def test_product_never_imports_oracle():
    pkg = ROOT / "paper_conf_ipps_hellwigcmbw23_b200"
    for p in list(pkg.rglob("*.py")) + list(pkg.rglob("*.cu")) + list(pkg.rglob("*.cuh")) + \
            list(pkg.rglob("*.h")) + [HEADER]:
        txt = p.read_text()
        assert "import oracle" not in txt and "from oracle" not in txt, p
        assert "cd_oracle" not in txt and "liborc" not in txt, p


def test_plan_extra_p_models(cds):
    """cd_plan against PAPER.md Section IV-B as printed: Eq. 3 / Eq. 4, the
    capacity rule c = max(c', 10^4) * 2 * 2 and g_ch = 16 c, o = t / s_ps
    (with both window ends included, R4), p and r_c = o / p."""
    n, d = 64000, 2.0
    g = cds.plan(n, 0.0, 86400.0, 1.0, d, "grid", mem_bytes=24 << 30)
    # Eq. 3 with s = 1 s, t = 86400 s, d = 2 km: 2.32e-9 * 64000^2 * 86400 * 2^1.75
    assert g["est_candidates"] == pytest.approx(2.32e-9 * 4.096e9 * 86400.0 * 2.0 ** 1.75, rel=1e-12)
    assert g["samples"] == 86401
    assert g["capacity"] == pytest.approx(4 * g["est_candidates"], rel=1e-12)
    assert g["capacity_bytes"] == pytest.approx(16 * g["capacity"], rel=1e-12)
    assert g["est_candidates_per_step"] == pytest.approx(g["est_candidates"] / 86400.0, rel=1e-12)
    h = cds.plan(n, 0.0, 86400.0, 9.0, d, "hybrid", mem_bytes=24 << 30)
    # Eq. 4: 2.14e-9 n^2 s^(5/3) t d with s = 9 s
    assert h["est_candidates"] == pytest.approx(2.14e-9 * 4.096e9 * 9.0 ** (5 / 3) * 86400.0 * 2.0, rel=1e-12)
    assert h["samples"] == 9601
    # the 10^4 floor of P:272 for a tiny screen
    tiny = cds.plan(100, 0.0, 60.0, 1.0, 1.0, "grid", mem_bytes=1 << 30)
    assert tiny["est_candidates"] < 1e4 and tiny["capacity"] == 4e4
    # p and r_c as defined; p grows linearly with the free memory
    for m in (8 << 30, 24 << 30, 180 << 30):
        q = cds.plan(n, 0.0, 86400.0, 1.0, d, "grid", mem_bytes=m)
        assert q["grids_in_memory"] == pytest.approx((m - q["fixed_bytes"]) / q["bytes_per_grid"], rel=1e-12)
        assert q["rounds"] == pytest.approx(q["samples"] / q["grids_in_memory"], rel=1e-12)
    # n^2 scaling of both models (the paper's "mainly the product of n, t and d")
    g2 = cds.plan(2 * n, 0.0, 86400.0, 1.0, d, "grid", mem_bytes=24 << 30)
    assert g2["est_candidates"] == pytest.approx(4 * g["est_candidates"], rel=1e-12)
    with pytest.raises(cds.CdError):
        cds.plan(n, 10.0, 0.0, 1.0, d, "grid", mem_bytes=1 << 30)
