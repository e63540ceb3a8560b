"""C-ABI boundary checks that need no GPU: the library loads, exports every
function include/stemroot.h declares, and the Python binding's struct layouts
match the header (compiled with gcc)."""
import os
import re
import subprocess

import pytest

import paper_conf_micro_chungnkk25_b200 as sr

HEADER = sr.HEADER


@pytest.fixture(scope="module")
def lib():
    sr.build()
    return sr.lib()


def declared_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"STEM_API\s+[\w\s\*]+?\b(stem_\w+)\s*\(", src)))


def test_header_declares_the_abi():
    names = declared_functions()
    assert "stem_root_plan" in names and "stem_plan_free" in names
    assert set(names) == set(sr.EXPORTS)


def test_library_exports_every_declared_symbol(lib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", sr.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (stem_\w+)", out))
    for name in declared_functions():
        assert name in exported, name
        assert hasattr(lib, name)
    # nothing else leaks out of the shared object under the stem_ prefix
    assert exported == set(declared_functions())


def test_strerror_is_total(lib):
    for st in (0, -1, -2, -3, -4, -5, -6, -7, 12345):
        assert isinstance(sr.strerror(st), str) and sr.strerror(st)


def test_struct_layouts_match_header(tmp_path):
    import ctypes as C
    prog = tmp_path / "layout.c"
    structs = {"stem_trace": sr.stem_trace, "stem_opts": sr.stem_opts, "stem_cluster": sr.stem_cluster,
               "stem_plan": sr.stem_plan, "stem_device_plan": sr.stem_device_plan, "stem_stats": sr.stem_stats}
    lines = ['#include <stdio.h>', '#include <stddef.h>', f'#include "{HEADER}"', 'int main(void){']
    for s, cls in structs.items():
        lines.append(f'printf("{s} %zu\\n", sizeof({s}));')
        for f, _ in cls._fields_:
            lines.append(f'printf("{s}.{f} %zu\\n", offsetof({s}, {f}));')
    lines.append("return 0;}")
    prog.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-o", str(exe), str(prog)])
    got = dict(l.split() for l in subprocess.check_output([str(exe)]).decode().split("\n") if l)
    for s, cls in structs.items():
        assert int(got[s]) == C.sizeof(cls), s
        for f, _ in cls._fields_:
            assert int(got[f"{s}.{f}"]) == getattr(cls, f).offset, (s, f)


def test_product_path_has_no_oracle_dependency():
    root = os.path.dirname(sr.__file__)
    for dirpath, _, files in os.walk(root):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, fn)).read()
                for pat in ("import oracle", "from oracle", "liboracle", "stemroot_oracle", "or_plan"):
                    assert pat not in text, (fn, pat)


def test_binding_rejects_wrong_dtypes_and_shapes():
    """the binding must not reinterpret a wrong dtype's bytes
    (torch's default int64 ids, float32 times or metrics) -- it raises before
    any library call; numpy integer arrays of other widths are range-checked
    and converted, 4-byte ones viewed."""
    import numpy as np
    import torch
    k = np.zeros(8, np.uint32)
    t = np.arange(8, dtype=np.uint32)
    with pytest.raises(TypeError):
        sr._trace(torch.zeros(8, dtype=torch.int64), torch.zeros(8, dtype=torch.int32), 1, None)
    with pytest.raises(TypeError):
        sr._trace(torch.zeros(8, dtype=torch.int32), torch.zeros(8, dtype=torch.float32), 1, None)
    with pytest.raises(TypeError):
        sr._trace(torch.zeros(8, dtype=torch.int32), torch.zeros(8, dtype=torch.int32), 1,
                  torch.zeros((2, 8), dtype=torch.float32))
    with pytest.raises(TypeError):
        sr._trace(k, t.astype(np.float64), 1, None)
    with pytest.raises(ValueError):
        sr._trace(k, t[:7], 1, None)
    with pytest.raises(ValueError):
        sr._trace(k, t, 1, np.zeros((2, 7)))
    with pytest.raises(ValueError):
        sr._trace(k.astype(np.int64) - 1, t, 1, None)
    tr, dev, keep = sr._trace(k.astype(np.int64), t.astype(np.uint16), 1, np.ones((3, 8), np.float32))
    assert (tr.n, tr.n_metrics, dev) == (8, 3, -1)
    assert keep[0].dtype == np.uint32 and keep[1].dtype == np.uint32 and keep[2].dtype == np.float64
    tr, _, keep = sr._trace(k.view(np.int32), t, 1, np.ones(8))
    assert tr.n_metrics == 1 and keep[0].dtype == np.uint32
