"""CPU-side checks of the C-ABI boundary: the library builds, loads and exports every function
declared in include/gsnp.h; the record layout is 40 bytes on both sides of the ABI."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess
import tempfile

import numpy as np

from paper_conf_icpp_luzlwfl11_b200 import build as gbuild
from paper_conf_icpp_luzlwfl11_b200 import gsnp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "gsnp.h")


def _declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gsnp_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    gbuild.build()
    L = ctypes.CDLL(gbuild.LIB)
    decl = _declared()
    assert len(decl) >= 12
    for name in decl:
        assert hasattr(L, name), name
    assert sorted(gsnp.SYMBOLS) == decl
    out = subprocess.run(["nm", "-D", "--defined-only", gbuild.LIB], capture_output=True,
                         text=True).stdout
    for name in decl:
        assert re.search(rf"\bT {name}\b", out), name


def test_params_default_and_strerror_without_gpu():
    p = gsnp.params_default()
    assert p.abi_version == 1 and p.max_read_len == 100 and p.q_max == 40
    assert p.het_novel == 1e-3 and p.althom_novel == 5e-4
    assert p.global_dep == 0.9 and p.pcr_dep == 0.5 and p.flags == gsnp.GSNP_RANK_SUM
    assert gsnp.lib().gsnp_strerror(-3) == b"reads not sorted by position"
    assert gsnp.lib().gsnp_last_error(None) == b""
    assert gsnp.lib().gsnp_launch_count(None) == 0


def test_record_layout_matches_header():
    prog = r'''
#include <stddef.h>
#include <stdio.h>
#include "gsnp.h"
int main(void) {
  printf("%zu %zu %zu %zu %zu %zu %zu\n", sizeof(gsnp_record), offsetof(gsnp_record, ref),
         offsetof(gsnp_record, cnt_uni1), offsetof(gsnp_record, depth),
         offsetof(gsnp_record, rank_p), offsetof(gsnp_record, post1), sizeof(gsnp_params));
  return 0;
}
'''
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "t.c")
        open(c, "w").write(prog)
        exe = os.path.join(d, "t")
        subprocess.check_call(["gcc", "-I" + os.path.join(ROOT, "include"), "-o", exe, c])
        vals = [int(x) for x in subprocess.check_output([exe]).split()]
    dt = gsnp.RECORD_DTYPE
    assert vals[:6] == [40, dt.fields["ref"][1], dt.fields["cnt_uni1"][1], dt.fields["depth"][1],
                        dt.fields["rank_p"][1], dt.fields["post1"][1]]
    assert vals[6] == ctypes.sizeof(gsnp.gsnp_params)


def test_create_without_gpu_reports_cuda_error():
    import torch
    if torch.cuda.is_available():
        return
    ref = np.zeros(100, np.uint8)
    try:
        gsnp.Context(ref)
    except gsnp.GsnpError as e:
        assert e.status in (-6, -1)
    else:  # pragma: no cover
        raise AssertionError("expected an error without a GPU")


def test_oracle_and_product_share_no_code():
    """The oracle and the CUDA path are independent (no imports either way)."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_luzlwfl11_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dp, f)).read()
                assert "import oracle" not in s and "from oracle" not in s and "oracle.c" not in s, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            s = open(os.path.join(ROOT, "oracle", f)).read()
            assert not re.search(r"^\s*(import|from)\s+paper_conf_icpp_luzlwfl11_b200", s, re.M)
            assert not re.search(r"^\s*#\s*include\s*[<\"].*gsnp", s, re.M)
            assert not re.search(r"CDLL\([^)]*gsnp", s)
