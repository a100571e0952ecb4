"""CPU-only checks of the C-ABI library: it loads, exports every symbol that
include/griffin.h declares, and its pure-host helpers (shard ranges, the
merge-path split used by the device partitioner) match the paper's examples.
No compute call that needs a GPU is made here."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_ppopp_0044ws18_b200 as g
from conftest import ROOT, read_golden
from helpers import corpus_from_lists

HEADER = os.path.join(ROOT, "include", "griffin.h")


def _declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(griffin_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = g.load_library()
    syms = _declared_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(lib, s), s
    out = subprocess.run(["nm", "-D", "--defined-only", g.LIB_PATH], capture_output=True,
                         text=True).stdout
    exported = set(re.findall(r" T (griffin_\w+)", out))
    assert set(syms) <= exported


def test_library_is_sm100a():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", g.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_shard_ranges_partition_docids():
    for N in [1, 7, 100, 1_000_003]:
        for G in [1, 2, 3, 4, 8]:
            prev = 0
            for s in range(G):
                a, b = g.griffin_shard_range(N, G, s)
                assert a == prev and a <= b
                per = -(-N // G)
                assert a == min(N, s * per) and b == min(N, (s + 1) * per)
                prev = b
            assert prev == N
    with pytest.raises(g.GriffinError):
        g.griffin_shard_range(10, 9, 0)


def test_merge_path_fig6_splits():
    """Fig. 6: p = 4 diagonals give splits (0,0),(2,2),(5,3),(7,5),(9,7)."""
    gd = read_golden("merge_path_fig6.txt")
    A = [int(x) for x in gd["A"][0]]
    B = [int(x) for x in gd["B"][0]]
    p = int(gd["p"][0][0])
    want = [int(x) for x in gd["splits"][0]]
    want = list(zip(want[0::2], want[1::2]))
    step = (len(A) + len(B)) // p
    got = [g.griffin_merge_path_split(A, B, d * step, fixup=True) for d in range(p + 1)]
    assert got == want
    # each partition merged on its own yields the paper's intersection (1,3,7,25,31)
    res = []
    for (i0, j0), (i1, j1) in zip(got[:-1], got[1:]):
        res += sorted(set(A[i0:i1]) & set(B[j0:j1]))
    assert res == [int(x) for x in gd["result"][0]]


def test_merge_path_tie_fixup():
    """without the fix-up, diagonal 7 splits the matched pair (7,7)
    as (5,2); with it the split is (5,3) and no matched pair is ever split."""
    gd = read_golden("merge_path_fig6.txt")
    A = [int(x) for x in gd["A"][0]]
    B = [int(x) for x in gd["B"][0]]
    assert g.griffin_merge_path_split(A, B, 7, fixup=False) == (5, 2)
    assert g.griffin_merge_path_split(A, B, 7, fixup=True) == (5, 3)
    for d in range(len(A) + len(B) + 1):
        i, j = g.griffin_merge_path_split(A, B, d, fixup=True)
        assert not (i > 0 and j < len(B) and A[i - 1] == B[j])


def test_merge_path_partitions_bruteforce():
    """Random sorted sets, every p: per-partition intersections concatenate to
    the full intersection, and partitions are balanced to within one element
    (P:716-719)."""
    rng = np.random.default_rng(3)
    for _ in range(200):
        A = np.sort(rng.choice(300, size=int(rng.integers(0, 80)), replace=False))
        B = np.sort(rng.choice(300, size=int(rng.integers(0, 80)), replace=False))
        tot = len(A) + len(B)
        p = int(rng.integers(1, 12))
        diags = [min(tot, (tot * s + p - 1) // p) for s in range(p + 1)]
        sp = [g.griffin_merge_path_split(A, B, d, True) for d in diags]
        res = []
        for (i0, j0), (i1, j1) in zip(sp[:-1], sp[1:]):
            assert i0 <= i1 and j0 <= j1
            assert abs((i1 - i0) + (j1 - j0) - (diags[1] - diags[0])) <= 2 or p == 1
            res += sorted(set(A[i0:i1].tolist()) & set(B[j0:j1].tolist()))
        assert res == sorted(set(A.tolist()) & set(B.tolist()))


def test_build_without_gpu_fails_loudly():
    """No CPU fallback: with no CUDA device the build returns an error."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    c = corpus_from_lists(10, [[1, 2, 3]])
    with pytest.raises(g.GriffinError) as e:
        g.GriffinIndex(c)
    assert e.value.status in (6, 4)


def test_invalid_arguments_rejected_on_host():
    with pytest.raises(g.GriffinError):
        g.griffin_merge_path_split([1, 2], [3], 9)


def test_multi_gpu_options_rejected_on_host():
    """num_gpus / exchange are checked before any device is touched (§8(b))."""
    c = corpus_from_lists(10, [[1, 2, 3]])
    with pytest.raises(g.GriffinError) as e:
        g.GriffinIndex(c, num_gpus=9)
    assert e.value.status == 1
    with pytest.raises(g.GriffinError) as e:
        g.GriffinIndex(c, num_gpus=2, exchange=7)
    assert e.value.status == 1
    with pytest.raises(g.GriffinError) as e:   # a multi handle builds its shards itself
        g.GriffinIndex(c, num_gpus=2, num_shards=2)
    assert e.value.status == 1


def test_profile_struct_layout_matches_header(tmp_path):
    """The binding's ctypes mirror of griffin_profile has the C struct's size
    and field offsets (compiled from include/griffin.h with the host gcc)."""
    fields = [f for f, _ in g.Profile._fields_]
    src = tmp_path / "layout.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "griffin.h"\n'
                   'int main(void) {\n  printf("%zu\\n", sizeof(griffin_profile));\n' +
                   "".join(f'  printf("%zu\\n", offsetof(griffin_profile, {f}));\n' for f in fields) +
                   "  return 0;\n}\n")
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)],
                   check=True)
    out = [int(x) for x in subprocess.run([str(exe)], capture_output=True, text=True,
                                          check=True).stdout.split()]
    assert out[0] == ctypes.sizeof(g.Profile)
    assert out[1:] == [getattr(g.Profile, f).offset for f in fields]
