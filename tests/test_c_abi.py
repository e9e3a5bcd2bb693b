"""The C ABI from plain C (tests/c_abi_example.c): the header compiles as C11 and the program
links against libcdscreen.so; without a GPU every compute call reports CD_ENODEV; on a B200 its
result equals the Python binding's, record for record."""
import os
import subprocess
from pathlib import Path

import numpy as np
import pytest

ROOT = Path(__file__).resolve().parent.parent
PKG = ROOT / "paper_conf_ipps_hellwigcmbw23_b200"


def _build_example(tmp_path):
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    cds.lib()   # built in-tree
    exe = tmp_path / "c_abi_example"
    cmd = ["gcc", "-std=c11", "-O2", "-Wall", "-Werror", f"-I{ROOT / 'include'}",
           str(ROOT / "tests" / "c_abi_example.c"), f"-L{PKG}", "-l:libcdscreen.so",
           f"-Wl,-rpath,{PKG}", "-o", str(exe)]
    subprocess.run(cmd, check=True)
    return exe


def _write_pop(pop, path):
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    np.concatenate([np.asarray(pop[k], dtype=np.float64) for k in cds.FIELDS]).tofile(path)


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.mark.skipif(_has_gpu(), reason="checks the no-GPU behaviour")
def test_c_example_builds_and_reports_no_device(tmp_path):
    from tools import popgen
    exe = _build_example(tmp_path)
    pop = popgen.random_population(100, 3)
    _write_pop(pop, tmp_path / "pop.f64")
    r = subprocess.run([str(exe), str(tmp_path / "pop.f64"), "100", "0", "60", "1", "5", "0",
                        str(tmp_path / "out.bin")], capture_output=True, text=True)
    assert r.returncode == 1 and "CD_ENODEV" in r.stderr, (r.returncode, r.stderr)


@pytest.mark.gpu
@pytest.mark.parametrize("mode,dt", [(0, 1.0), (1, 9.0)])
def test_c_example_matches_binding(tmp_path, mode, dt):
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    exe = _build_example(tmp_path)
    pop, cfg, _ = popgen.make_config(1)
    n = len(pop["a"])
    _write_pop(pop, tmp_path / "pop.f64")
    r = subprocess.run([str(exe), str(tmp_path / "pop.f64"), str(n), str(cfg.t0), str(cfg.t1), str(dt),
                        str(cfg.d), str(mode), str(tmp_path / "out.bin")], capture_output=True, text=True,
                       env=dict(os.environ))
    assert r.returncode == 0, r.stderr
    raw = (tmp_path / "out.bin").read_bytes()
    cnt = int(np.frombuffer(raw[:8], dtype="<u8")[0])
    got = np.frombuffer(raw[8:], dtype=cds.CONJ_DTYPE)
    want = cds.screen(pop, cfg.t0, cfg.t1, dt, cfg.d, mode="grid" if mode == 0 else "hybrid")
    assert cnt == len(want) > 0
    assert np.array_equal(got, want)
