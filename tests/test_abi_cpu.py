"""CPU-only checks of the C ABI library: it loads, exports every symbol frugal.h
declares, and validates configs without touching a GPU."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _lib():
    from paper_conf_asplos_xiezggl25_b200 import build as B
    B.build()
    from paper_conf_asplos_xiezggl25_b200 import frugal as F
    return F


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "frugal.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(frugal_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    F = _lib()
    L = F.lib()
    syms = declared_symbols()
    assert len(syms) >= 15
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing, missing
    assert set(syms) == set(F.EXPORTED)


def test_sass_is_sm100a():
    import subprocess
    F = _lib()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", F.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


@pytest.mark.parametrize("field,value", [("world", 0), ("dim", 6), ("lookahead", 1), ("lookahead", 40),
                                         ("age_out", 0), ("n_rows", 0), ("batch", 0), ("opt", 7)])
def test_config_validation(field, value):
    F = _lib()
    cfg = F.Config(world=1, rank=0, device=0, dim=16, n_rows=100, slots=1, batch=4, lookahead=4, age_out=2,
                   opt=1, lr=0.1, eps=1e-10, init_accum=0.0, init_scale=0.05, init_seed=3, hot_ids=None,
                   n_hot=0, shm_name=None, mode=0, flags=0)
    setattr(cfg, field, value)
    h = C.c_void_p()
    st = F.lib().frugal_init(C.byref(cfg), C.byref(h))
    assert st == -1, F.lib().frugal_last_error()
    assert not h.value


def test_world_gt1_needs_shm():
    F = _lib()
    cfg = F.Config(world=2, rank=0, device=0, dim=16, n_rows=100, slots=1, batch=4, lookahead=4, age_out=2,
                   opt=1, lr=0.1, eps=1e-10, init_accum=0.0, init_scale=0.05, init_seed=3, hot_ids=None,
                   n_hot=0, shm_name=None, mode=0, flags=0)
    h = C.c_void_p()
    assert F.lib().frugal_init(C.byref(cfg), C.byref(h)) == -1
    assert b"shm" in F.lib().frugal_last_error()


def test_world_gt1_needs_run_nonce():
    """A shared table needs a run nonce (ranks > 0 attach only to their run's segment)."""
    F = _lib()
    cfg = F.Config(world=2, rank=1, device=0, dim=16, n_rows=100, slots=1, batch=4, lookahead=4, age_out=2,
                   opt=1, lr=0.1, eps=1e-10, init_accum=0.0, init_scale=0.05, init_seed=3, hot_ids=None,
                   n_hot=0, shm_name=b"/frugal_nonce_test", mode=0, flags=0, run_nonce=0)
    h = C.c_void_p()
    assert F.lib().frugal_init(C.byref(cfg), C.byref(h)) == -1
    assert b"run_nonce" in F.lib().frugal_last_error()
    assert not h.value


def test_null_ctx_calls_fail_cleanly():
    F = _lib()
    L = F.lib()
    assert L.frugal_step(None, 0, None, None, None) == -1
    assert L.frugal_lookup(None, 0, None, None) == -1
    assert L.frugal_destroy(None) == 0


def test_product_path_does_not_import_oracle():
    """The product (package + CUDA sources) never imports, links or loads oracle/."""
    pkg = os.path.join(ROOT, "paper_conf_asplos_xiezggl25_b200")
    pat = re.compile(r"^\s*(from\s+oracle|import\s+oracle)|liboracle|frugal_oracle", re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                assert not pat.search(open(os.path.join(dirpath, f)).read()), f


def test_bench_module_imports_and_parses():
    """bench.py must at least import and parse its arguments without a GPU."""
    import importlib
    import sys
    sys.argv = ["bench.py"]
    b = importlib.import_module("bench")
    a = b.parse()
    assert a.gpus == 1 and a.warmup >= 3 and a.exchange == "host"
    assert b.dist_max(3.0, 1) == 3.0


@pytest.mark.parametrize("n_order", [-1, 5, 101])
def test_host_order_validation(n_order):
    """frugal_config.host_order: a negative or too long count, or a count without a list,
    is rejected before any device work."""
    F = _lib()
    cfg = F.Config(world=1, rank=0, device=0, dim=16, n_rows=100, slots=1, batch=4, lookahead=4, age_out=2,
                   opt=1, lr=0.1, eps=1e-10, init_accum=0.0, init_scale=0.05, init_seed=3, hot_ids=None,
                   n_hot=0, shm_name=None, mode=0, flags=0, host_order=None, n_order=n_order)
    h = C.c_void_p()
    assert F.lib().frugal_init(C.byref(cfg), C.byref(h)) == -1
    assert not h.value


def test_workload_host_order():
    """The frequency layout of past traffic: distinct seen rows, most frequent first, ties by id."""
    import numpy as np
    from paper_conf_asplos_xiezggl25_b200 import workload as W
    cfg = W.config("tiny", world=2, batch=64)
    st = W.gen_stream(cfg, 8)
    o = W.host_order(cfg, st.ids, st.counts)
    freq = np.bincount(st.ids.ravel(), minlength=cfg.n_rows)
    assert len(set(o.tolist())) == len(o) == int((freq > 0).sum())
    key = [(-int(freq[k]), int(k)) for k in o]
    assert key == sorted(key)


@pytest.mark.parametrize("cname,pyname", [("frugal_config", "Config"), ("frugal_schedule_info", "ScheduleInfo"),
                                          ("frugal_stats", "Stats")])
def test_struct_layouts_match_header(cname, pyname, tmp_path):
    """The ctypes mirrors of the ABI structs have the C compiler's size and field offsets
    (a field appended to frugal.h but not to frugal.py -- or vice versa -- would make the
    library write past, or read garbage from, the binding's buffer)."""
    import subprocess
    F = _lib()
    py = getattr(F, pyname)
    fields = [f[0] for f in py._fields_]
    prog = ["#include <stdio.h>", "#include <stddef.h>", '#include "frugal.h"', "int main(void) {",
            f'  printf("%zu\\n", sizeof({cname}));']
    prog += [f'  printf("%zu\\n", offsetof({cname}, {f}));' for f in fields]
    prog += ["  return 0;", "}"]
    src = tmp_path / "layout.c"
    src.write_text("\n".join(prog) + "\n")
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = [int(x) for x in subprocess.check_output([str(exe)]).split()]
    assert got[0] == C.sizeof(py), (cname, got[0], C.sizeof(py))
    for f, off in zip(fields, got[1:]):
        assert getattr(py, f).offset == off, (cname, f, off, getattr(py, f).offset)
