"""CPU-only checks of the C-ABI library (no GPU calls): it loads, exports every symbol include/lsqr_avugsr.h
declares, its host-side integer helpers (obs-per-star, constraint rows, shard map) are bit-exact with the oracle's
O-GEN/O-SHARD, and argument validation fails with LSQR_EINVAL before touching the device."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import oracle
import workloads as W
from paper_conf_sc_malenzacsbvba24_b200 import _capi
import paper_conf_sc_malenzacsbvba24_b200 as avu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = []
    for fn in os.listdir(os.path.join(ROOT, "include")):
        if fn.endswith(".h"):
            src = open(os.path.join(ROOT, "include", fn)).read()
            src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
            names += re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\*?\s*(lsqr_[a-z0-9_]+)\s*\(", src,
                                flags=re.M)
    return sorted(set(names))


def test_library_exports_every_declared_symbol():
    L = _capi.lib()
    names = declared_functions()
    assert len(names) >= 25, names
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(_capi.EXPORTS), set(names) ^ set(_capi.EXPORTS)
    assert L.lsqr_abi_version() == 2
    assert L.lsqr_strerror(-6) == b"rows not grouped by star / inconsistent with obs_per_star"


@pytest.mark.parametrize("w", [W.C1, W.C2, W.micro(), W.micro(n_stars=5, obs=1, jitter=50),
                               W.Workload("odd", n_stars=1001, n_obs=100_007, n_att=30, n_instr=12, jitter_pct=37,
                                          seed=99)])
def test_obs_per_star_bit_exact(w):
    a = avu.synth_obs_per_star(w.seed, w.n_stars, w.n_obs, w.jitter_pct)
    b = oracle.star_counts(w)
    assert np.array_equal(a, b)


@pytest.mark.parametrize("w", [W.C1C, W.C2, W.micro(n_stars=9, obs=20, n_ext=4, seed=9)])
def test_constraints_bit_exact(w):
    a = avu.synth_constraints(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_ext_stars)
    b = oracle.constraints(w)
    for x, y in zip(a, b):
        assert x.dtype == y.dtype and np.array_equal(x.view(np.uint8), y.view(np.uint8))


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_shard_map_bit_exact(P):
    for w in (W.C2, W.C4.replace(n_stars=400_000, n_obs=78_000_000), W.micro(n_stars=11, obs=3)):
        counts = oracle.star_counts(w)
        a = avu.shard_map(counts, w.n_obs, P)
        b = oracle.shard(oracle.row_ptr(counts), w.n_obs, P)
        assert np.array_equal(a, b)


def test_create_rejects_bad_arguments_without_gpu():
    L = _capi.lib()
    env = _capi.Env()
    env.rank, env.nranks = 0, 1
    h = C.c_void_p(1234)
    # n_att not a multiple of 3 / n_glob out of range / bad rank / nranks>1 without an NCCL id
    assert L.lsqr_create(10, 100, 31, 12, 1, None, None, C.byref(env), C.byref(h)) == -1
    assert h.value is None
    assert L.lsqr_create(10, 100, 30, 12, 2, None, None, C.byref(env), C.byref(h)) == -1
    env2 = _capi.Env(); env2.rank, env2.nranks = 2, 2
    assert L.lsqr_create(10, 100, 30, 12, 1, None, None, C.byref(env2), C.byref(h)) == -1
    env3 = _capi.Env(); env3.rank, env3.nranks = 0, 2
    assert L.lsqr_create(10, 100, 30, 12, 1, None, None, C.byref(env3), C.byref(h)) == -1
    bad_counts = np.array([5] * 10, dtype=np.int64)  # sums to 50 != 100
    assert L.lsqr_create(10, 100, 30, 12, 1, bad_counts.ctypes.data_as(C.c_void_p), None, C.byref(env),
                         C.byref(h)) == -1
    ptr = np.array([0, 1], dtype=np.int64); col = np.array([10 ** 9], dtype=np.int64); val = np.ones(1)
    cs = _capi.Constraints(1, ptr.ctypes.data, col.ctypes.data, val.ctypes.data, None)
    assert L.lsqr_create(10, 100, 30, 12, 1, None, C.byref(cs), C.byref(env), C.byref(h)) == -1
    # host helpers validate too
    assert L.lsqr_synth_obs_per_star(1, 0, 10, 0, None) == -1
    assert L.lsqr_synth_constraints(1, 10, 30, 7, 5, None, None, None) == -1
    assert L.lsqr_destroy(None) == 0


def test_missing_extension_fails_loudly(monkeypatch, tmp_path):
    """No CPU fallback: without the shared library every entry point raises (the binding never computes)."""
    from paper_conf_sc_malenzacsbvba24_b200 import _capi, build as _build
    monkeypatch.setattr(_build, "LIB", str(tmp_path / "liblsqr_avugsr.so"))
    monkeypatch.setattr(_capi, "_lib", None)
    with pytest.raises(RuntimeError, match="missing"):
        _capi.lib(build_if_missing=False)


def test_stale_library_is_refused(monkeypatch):
    """The library embeds the hash of the sources it was built from (lsqr_build_id); a library built from other
    sources is rebuilt (needs_build) or, when building is not allowed, refused -- never loaded silently."""
    from paper_conf_sc_malenzacsbvba24_b200 import _capi, build as _build
    L = _capi.lib()
    assert L.lsqr_build_id().decode() == _build.source_hash() == _build.built_id()
    assert not _build.needs_build()
    monkeypatch.setattr(_build, "source_hash", lambda: "f" * 16)  # as if a source had changed since the build
    assert _build.needs_build()
    monkeypatch.setattr(_capi, "_lib", None)
    with pytest.raises(RuntimeError, match="other sources"):
        _capi.lib(build_if_missing=False)


def test_product_package_never_touches_the_oracle():
    """The product path (package sources, CUDA, C ABI header) shares no code with oracle/ and does not import it."""
    import glob
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    files = glob.glob(os.path.join(root, "paper_conf_sc_malenzacsbvba24_b200", "**", "*.*"), recursive=True)
    files += glob.glob(os.path.join(root, "include", "*.h"))
    srcs = [f for f in files if f.endswith((".py", ".cu", ".cuh", ".h", ".c", ".cpp"))]
    assert srcs
    for f in srcs:
        txt = open(f, encoding="utf-8", errors="replace").read()
        for bad in ("import oracle", "from oracle", "avugsr_oracle", "orc_"):
            assert bad not in txt, (f, bad)
