"""CPU-side checks of the C-ABI boundary: the library loads, exports every symbol include/kgs.h
declares, and fails loudly (no CPU fallback) when no GPU is present."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "kgs.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(kgs_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("kgs_load_graph", "kgs_query", "kgs_query_device", "kgs_query_fetch", "kgs_result_answer",
                 "kgs_result_levels", "kgs_result_centrals", "kgs_result_stats", "kgs_free_graph"):
        assert must in names


def test_library_exports_every_declared_symbol():
    import paper_conf_icde_yangajtw19_b200 as kgs
    L = kgs.lib()
    for name in _declared():
        assert hasattr(L, name), name
    assert set(kgs.EXPORTED) == set(_declared())
    assert "sm_100a" in kgs.kgs_version()


def test_params_default_match_paper():
    import paper_conf_icde_yangajtw19_b200 as kgs
    p = kgs.kgs_params_default()
    assert p.alpha == 0.1 and p.lambda_ == 0.2          # Table III
    assert p.max_depth == 254 and p.block_central == 1 and p.level_cover == 1


def test_struct_layout_matches_header(tmp_path):
    """The ctypes mirrors have the C compiler's size and field offsets for every struct in kgs.h."""
    import subprocess
    import paper_conf_icde_yangajtw19_b200 as kgs
    structs = [kgs.kgs_graph_desc, kgs.kgs_params, kgs.kgs_answer, kgs.kgs_stats, kgs.kgs_vp_buffers]
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "kgs.h"', "int main(void) {"]
    for st in structs:
        nm = st.__name__
        lines.append(f'printf("{nm} %zu\\n", sizeof({nm}));')
        for f, _ in st._fields_:
            cf = "lambda" if f == "lambda_" else f
            lines.append(f'printf("{nm}.{f} %zu\\n", offsetof({nm}, {cf}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include")
    subprocess.run(["gcc", "-I", inc, str(src), "-o", str(exe)], check=True)
    got = dict(l.split() for l in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split("\n") if l)
    for st in structs:
        nm = st.__name__
        assert int(got[nm]) == ctypes.sizeof(st), nm
        for f, _ in st._fields_:
            assert int(got[f"{nm}.{f}"]) == getattr(st, f).offset, (nm, f)


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_icde_yangajtw19_b200 as kgs
    import synth
    g = synth.from_edges(3, [(0, 1), (1, 2)], [0, 0, 0], [[0], [2]], 2.0)
    with pytest.raises(kgs.KgsError) as ei:
        kgs.kgs_load_graph(g)
    assert ei.value.status == kgs.KGS_ECUDA


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_yangajtw19_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, re.M), f
                assert "liboracle" not in txt and "oracle.h" not in txt, f
