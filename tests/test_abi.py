"""CPU-side checks of the C-ABI library: it loads and exports every symbol include/ggrid.h
declares (no GPU compute calls here), plus pure host helpers."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def gg():
    from paper_conf_icde_li0qhdy18_b200 import build

    build.build()
    import paper_conf_icde_li0qhdy18_b200 as m

    return m


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "ggrid.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ggrid_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol(gg):
    names = _declared_functions()
    assert "ggrid_build" in names and "ggrid_ingest" in names and "ggrid_knn" in names
    L = ctypes.CDLL(gg.LIB_PATH)
    for n in names:
        assert hasattr(L, n), n
    assert sorted(gg.EXPORTS) == names


def test_struct_layouts_match_header(gg, tmp_path):
    """Every struct of include/ggrid.h: the C compiler's size and field offsets (gcc on the
    header itself) equal the ctypes mirror of the binding."""
    import subprocess

    structs = {"ggrid_graph": gg.ggrid_graph, "ggrid_opts": gg.ggrid_opts, "ggrid_stats_t": gg.ggrid_stats_t,
               "ggrid_prior_art_result": gg.ggrid_prior_art_result,
               "ggrid_prior_art_knn_result": gg.ggrid_prior_art_knn_result}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "ggrid.h"', "int main(void) {"]
    for name, cls in structs.items():
        lines.append(f'  printf("{name} %zu\\n", sizeof({name}));')
        for f, _ in cls._fields_:
            lines.append(f'  printf("{name}.{f} %zu\\n", offsetof({name}, {f}));')
    lines += ["  return 0;", "}"]
    c = tmp_path / "layout.c"
    c.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(c), "-o", str(exe)])
    got = dict(l.split() for l in subprocess.check_output([str(exe)], text=True).splitlines())
    for name, cls in structs.items():
        assert int(got[name]) == ctypes.sizeof(cls), name
        for f, _ in cls._fields_:
            assert int(got[f"{name}.{f}"]) == getattr(cls, f).offset, f"{name}.{f}"


def test_zvalue_worked_example(gg):
    # P@13347-13521: cell (3,4) -> 37 = (100101)_2, interleaving y=4 above x=3
    assert gg.ggrid_zvalue(3, 4) == 37
    assert gg.ggrid_zvalue(0, 0) == 0
    assert gg.ggrid_zvalue(1, 0) == 1 and gg.ggrid_zvalue(0, 1) == 2
    assert gg.ggrid_zvalue(0xFFFFFFFF, 0xFFFFFFFF) == (1 << 64) - 1


def test_strerror_and_version(gg):
    assert gg.strerror(0) == "ok"
    assert gg.strerror(-1) == "invalid argument"
    assert "sm_100a" in gg.ggrid_version()


def test_build_rejects_bad_graph_without_gpu_work(gg):
    import numpy as np

    # validation happens before any device call
    bad = dict(n_vertices=2, src=np.array([0], np.uint32), dst=np.array([5], np.uint32), w=np.array([1], np.uint32))
    with pytest.raises(gg.GGridError) as e:
        gg.ggrid_build(bad, 4)
    assert e.value.rc == gg.GGRID_EINVAL
    zero_w = dict(n_vertices=2, src=np.array([0], np.uint32), dst=np.array([1], np.uint32), w=np.array([0], np.uint32))
    with pytest.raises(gg.GGridError):
        gg.ggrid_build(zero_w, 4)
    ok = dict(n_vertices=2, src=np.array([0], np.uint32), dst=np.array([1], np.uint32), w=np.array([3], np.uint32))
    with pytest.raises(gg.GGridError):
        gg.ggrid_build(ok, 0)  # cell_size = 0


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_li0qhdy18_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "oracle.cpp" not in txt, f
