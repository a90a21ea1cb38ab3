"""C-ABI library checks that run without a GPU: the library loads, exports every
symbol include/gnn_sparse.h declares, and its host-only entry points (shards) match
the oracle bit-exactly.  No compute call is made here."""
import ctypes
import os
import re

import numpy as np
import pytest

import gen
import oracle
import paper_conf_ipps_fanwc23_b200 as gs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "gnn_sparse.h")).read()
    return sorted(set(re.findall(r"GNN_API[^;{]*?\b(gnn_\w+)\s*\(", src, re.S)))


def test_library_exports_every_declared_symbol():
    L = gs.lib()
    syms = declared_symbols()
    assert len(syms) >= 13
    for s in syms:
        assert hasattr(L, s), f"missing export {s}"
    assert sorted(gs.EXPORTS) == syms


def test_only_abi_symbols_are_exported():
    out = os.popen(f"nm -D --defined-only {gs.LIB_PATH}").read()
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    ours = {s for s in exported if s.startswith("gnn")}
    assert ours == set(declared_symbols())


def test_version_and_error_string():
    L = gs.lib()
    assert b"sm_100a" in L.gnn_version()
    assert isinstance(L.gnn_last_error(), bytes)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_shard_rows_matches_oracle(P):
    g = gen.powerlaw_graph(5000, 80000, gamma=2.2, n_comm=5, seed=50)
    assert np.array_equal(gs.shard_rows(g.row_ptr, P), oracle.shard_rows(g.row_ptr, P))
    sub = g.row_ptr[100:2001]  # a sub-view (row_ptr[0] != 0)
    assert np.array_equal(gs.shard_rows(sub, P), oracle.shard_rows(sub, P))


@pytest.mark.parametrize("nnz,P", [(0, 4), (10, 3), (114_848_857, 8), (7, 8), (2**31 - 1, 7)])
def test_shard_edges_matches_oracle(nnz, P):
    assert np.array_equal(gs.shard_edges(nnz, P), oracle.shard_edges(nnz, P))


def test_shard_bad_args_raise():
    with pytest.raises(gs.GnnError):
        gs.shard_edges(10, 0)
    with pytest.raises(gs.GnnError):
        gs.shard_rows(np.zeros(3, np.int32), 0)


def test_header_is_plain_c():
    """The ABI header compiles as C99 with no CUDA or torch headers."""
    rc = os.system(f"echo '#include \"gnn_sparse.h\"\nint main(void){{return 0;}}' | "
                   f"/usr/bin/gcc -std=c99 -Wall -Werror -I{ROOT}/include -x c - -o /dev/null")
    assert rc == 0


def test_binding_struct_layouts_match_header(tmp_path):
    """The ctypes mirrors of the ABI structs have the header's size and field offsets
    (a field added to gnn_plan_opts_t / gnn_plan_info_t must be added to the binding)."""
    structs = {"gnn_plan_opts_t": gs.PlanOpts, "gnn_plan_info_t": gs._PlanInfo,
               "gnn_graph_t": gs._Graph, "gnn_reorder_opts_t": gs.ReorderOpts}
    lines = ["#include <stdio.h>", "#include <stddef.h>", '#include "gnn_sparse.h"',
             "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'printf("{cname} size %zu\\n", sizeof({cname}));')
        for fname, _ in py._fields_:
            lines.append(f'printf("{cname} {fname} %zu\\n", offsetof({cname}, {fname}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    assert os.system(f"/usr/bin/gcc -std=c99 -I{ROOT}/include {src} -o {exe}") == 0
    got = {}
    for line in os.popen(str(exe)).read().splitlines():
        c, f, v = line.split()
        got[(c, f)] = int(v)
    for cname, py in structs.items():
        assert got[(cname, "size")] == ctypes.sizeof(py), cname
        for fname, _ in py._fields_:
            assert got[(cname, fname)] == getattr(py, fname).offset, (cname, fname)
