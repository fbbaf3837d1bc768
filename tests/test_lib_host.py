"""Host-side checks of the C-ABI library (no GPU needed, ``-m "not gpu"``).

* libooo.so loads and exports every function include/ooo.h declares.
* The schedule the library issues (ooo_schedule_order) equals the oracle's
  transcription of Algorithm 2 for many (L, k) -- two
  independent implementations (C++ vs Python) of the same pseudocode.
* Argument validation returns the documented statuses without touching a GPU.
"""
import ctypes
import os
import re

import pytest

from oracle import schedule as S
from paper_conf_eurosys_ohlks22_b200 import _lib, configs, stack

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    if not os.path.exists(_lib.LIB_PATH):
        from paper_conf_eurosys_ohlks22_b200 import build
        build.build()
    return _lib.load()


def test_library_exports_every_declared_symbol(lib):
    hdr = open(os.path.join(ROOT, "include", "ooo.h")).read()
    declared = set(re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(ooo_[a-z_0-9]+)\s*\(", hdr, re.M))
    assert len(declared) >= 20, declared
    for name in declared:
        assert hasattr(lib, name), name
    assert set(_lib.EXPORTS) == declared
    assert lib.ooo_abi_version() == 2


@pytest.mark.parametrize("L", [1, 2, 3, 5, 8, 13, 72, 144])
def test_library_schedule_equals_oracle_alg2(lib, L):
    for need in (False, True):
        assert stack.schedule_order(L, "in_order", 0, need) == S.in_order(L, need)
        for k in sorted({0, 1, 2, 3, L // 3, L // 2, L - 1, L, L + 5}):
            if k < 0:
                continue
            got = stack.schedule_order(L, "first_k", k, need)
            want = S.reverse_first_k(L, S.clamp_k(k, L), need, "paper")
            assert got == want, (L, k, need)
            assert S.is_valid_order(got, L, need)


def test_library_max_k_equals_oracle_reading(lib):
    import random
    rng = random.Random(3)
    for _ in range(200):
        L = rng.randint(1, 30)
        mdo = [rng.randint(0, 1000) for _ in range(L)]
        mdw = [rng.randint(0, 1000) for _ in range(L)]
        mf = rng.randint(0, 20000)
        mx = rng.randint(-5, 30000)
        assert stack.max_k(mf, mdo, mdw, mx) == S.max_k(mf, mdo, mdw, mx)


def test_invalid_arguments_are_rejected_without_gpu(lib):
    with pytest.raises(_lib.OooError) as e:
        stack.query_sizes([64, 100, 64], ["id", "id"], 32)          # width not a multiple of 64
    assert e.value.status == 2
    with pytest.raises(_lib.OooError) as e:
        stack.query_sizes([64, 64], ["id"], 12)                      # tokens % 8
    assert e.value.status == 2
    with pytest.raises(_lib.OooError) as e:
        stack.schedule_order(4, "first_k", -1)
    assert e.value.status == 1
    with pytest.raises(_lib.OooError) as e:
        stack.query_sizes([64, 64], [7], 32)                         # bad activation
    assert e.value.status == 1
    # create_stack with NULL pointers -> INVALID_ARGUMENT, nothing enqueued
    d, keep = stack._desc([64, 64], ["id"], 32, "bf16")
    h = ctypes.c_void_p()
    st = lib.ooo_create_stack(ctypes.byref(d), ctypes.byref(h))
    assert st == 1 and not h.value
    assert b"W/b" in lib.ooo_last_error()


def test_sizes_offsets_and_deferral_bytes(lib):
    c = configs.C2
    ws, gb = stack.query_sizes(c.dims, c.acts, c.tokens, "bf16")
    offs = stack.grad_offsets(c.dims, c.acts, c.tokens, "bf16")
    assert gb >= 2 * c.params() and gb < 2 * c.params() + 256
    # layers are contiguous: dW_i, db_i, dW_{i+1}, ...
    e = 0
    for i, (ow, ob) in enumerate(offs):
        assert ow == e and ob == e + c.dims[i] * c.dims[i + 1]
        e = ob + c.dims[i + 1]
    assert e == c.params()
    # activations + dZ stores dominate the workspace: at least X, dZ per layer
    need = sum(c.tokens * c.dims[i] * 2 for i in range(c.L)) + sum(c.tokens * d * 2 for d in c.dims[1:])
    assert ws >= need
    # memory cost of deferral (§3, E8): sum_{i=2..k} |dZ_i|
    for k in (0, 1, 2, 10, 72):
        want = sum(c.tokens * c.dims[i] * 2 for i in range(2, min(k, c.L) + 1))
        assert stack.deferral_bytes(c.dims, c.acts, c.tokens, "bf16", k) == want


def test_product_k_search_matches_oracle_reading():
    """The library's k search (``ooo_k_search``, regions.cpp; bench.py calls it
    with its measured throughput) and the oracle's transcription are
    independent implementations of the same reading (Q4): same
    best k and the same measurements in the same order."""
    import random
    from paper_conf_eurosys_ohlks22_b200.ksearch import search_k
    rng = random.Random(9)
    for L in (1, 2, 5, 10, 15, 24, 25, 35, 72, 144):
        for _ in range(20):
            vals = {k: rng.random() for k in range(L + 1)}
            kp, visited = search_k(L, lambda k: vals[k])
            vo = []
            ko = S.search_k(L, lambda k: vals[k], vo)
            assert kp == ko and visited == vo
            assert len(set(visited)) == len(visited)
        if L > 1:
            peak = rng.randint(0, L - 1)
            assert search_k(L, lambda k: -abs(k - peak))[0] == peak


def test_degenerate_sizes_without_gpu(lib):
    """Empty token batch -> UNSUPPORTED (nothing to compute, header: tokens >= 1);
    a one-layer stack's schedule is the lone dW_1 (dO_1 only with input grad)."""
    for t in (0, -8):
        with pytest.raises(_lib.OooError) as e:
            stack.query_sizes([64, 64], ["id"], t)
        assert e.value.status == 2
    for kind, k in [("in_order", 0), ("first_k", 0), ("first_k", 1), ("first_k", 5)]:
        assert stack.schedule_order(1, kind, k) == [-1]
        assert sorted(stack.schedule_order(1, kind, k, need_input_grad=True)) == [-1, 1]


def test_pipeline_host_validation(lib):
    """ooo_pipeline_* (cross-layer MP, §5.2.1): sizes and gradient offsets
    without a GPU; invalid groupings are rejected."""
    import ctypes
    from paper_conf_eurosys_ohlks22_b200 import stack
    dims, acts = [256] * 13, ["id"] * 12
    d = _lib.PipelineDesc()
    keep = (stack._i32arr(dims), stack._i32arr([0] * 12))
    d.num_layers, d.tokens, d.group_layers, d.n_stages, d.placement = 12, 64, 3, 2, 1
    d.world_size, d.rank = 1, 0
    d.dims = ctypes.cast(keep[0], ctypes.POINTER(ctypes.c_int32))
    d.acts = ctypes.cast(keep[1], ctypes.POINTER(ctypes.c_int32))
    ws, gb = ctypes.c_size_t(), ctypes.c_size_t()
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 0
    per_group = 3 * (256 * 256 + 256) * 2
    assert gb.value >= 4 * per_group
    offs = []
    for j in range(4):
        o = ctypes.c_int64()
        assert lib.ooo_pipeline_grads_offset(ctypes.byref(d), j, ctypes.byref(o)) == 0
        offs.append(o.value)
    assert offs == sorted(offs) and all(b - a >= per_group for a, b in zip(offs, offs[1:]))
    d.group_layers = 5                     # does not divide 12
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 1
    d.group_layers, d.n_stages = 3, 5      # more stages than groups
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 1
    d.n_stages, d.placement = 3, 0         # contiguous: stages must divide the groups
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 1
    # with a communicator (sizes need no NCCL): rank 0 of 2, modulo -> it owns groups 0 and 2 only
    uid = ctypes.create_string_buffer(128)
    d.n_stages, d.placement, d.world_size, d.rank = 2, 1, 2, 0
    d.nccl_unique_id = ctypes.cast(uid, ctypes.c_void_p)
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 0
    assert per_group * 2 <= gb.value < per_group * 3
    o = ctypes.c_int64()
    assert lib.ooo_pipeline_grads_offset(ctypes.byref(d), 2, ctypes.byref(o)) == 0
    assert lib.ooo_pipeline_grads_offset(ctypes.byref(d), 1, ctypes.byref(o)) == 1   # rank 1's group
    d.n_stages = 1                                  # one stage per rank required
    assert lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)) == 1
