"""CPU-side checks of the C-ABI boundary: the library loads and exports every entry point that
include/fastz.h declares; struct layouts seen by C match the binding's; bad arguments fail before any
device work.  No compute calls are made (no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_sc_gundaboluvt21_b200 import build, fastz

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "fastz.h")


def declared():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(fastz_[a-z_0-9]+)\s*\(", txt)))


def test_library_builds_and_exports_every_declared_symbol():
    path = build.build()
    L = ctypes.CDLL(path)
    names = declared()
    assert len(names) >= 10
    for n in names:
        assert hasattr(L, n), n
    assert sorted(fastz.EXPORTS) == names


def test_struct_layout_matches_header(tmp_path):
    src = tmp_path / "lay.c"
    src.write_text("""
#include <stdio.h>
#include <stddef.h>
#include "fastz.h"
int main(void){
 printf("%zu %zu %zu %zu %zu %zu %zu\\n", sizeof(fastz_alignment), sizeof(fastz_params), sizeof(fastz_seed),
        sizeof(fastz_stats), offsetof(fastz_alignment, cigar_off), offsetof(fastz_params, dev_alloc),
        offsetof(fastz_stats, bin_counts));
 return 0; }
""")
    exe = tmp_path / "lay"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)])
    vals = list(map(int, subprocess.check_output([str(exe)]).split()))
    assert vals == [fastz.ALIGN_DTYPE.itemsize, ctypes.sizeof(fastz.fastz_params), 16,
                    ctypes.sizeof(fastz.fastz_stats), fastz.ALIGN_DTYPE.fields["cigar_off"][1],
                    fastz.fastz_params.dev_alloc.offset, fastz.fastz_stats.bin_counts.offset]


def test_default_params_are_lastz_defaults():
    p = fastz.fastz_default_params()
    assert list(p.sub) == [91, -114, -31, -123, -114, 100, -125, -31, -31, -125, 100, -114, -123, -31, -114, 91]
    assert (p.gap_open, p.gap_extend, p.ydrop, p.gapped_threshold, p.eager_max) == (400, 30, 9400, 3000, 16)


@pytest.mark.parametrize("kw", [dict(gap_extend=0), dict(gap_open=-1), dict(ydrop=-5), dict(eager_max=17),
                                dict(eager_max=0), dict(sub=[40000] + [0] * 15)])
def test_bad_params_rejected_before_device_work(kw):
    p = fastz.fastz_default_params(**kw)
    with pytest.raises(fastz.FastzError) as ei:
        fastz.fastz_create(p, b"ACGT", b"ACGT", 0)
    assert ei.value.status == fastz.FASTZ_EINVAL


def test_strerror_and_destroy_null():
    L = fastz.lib()
    assert L.fastz_strerror(0) == b"ok"
    assert b"too small" in L.fastz_strerror(fastz.FASTZ_ETRUNC)
    L.fastz_destroy(None)


def test_sass_targets_sm100a_and_uses_the_integer_dp_instructions():
    """The library contains sm_100a SASS for every DP kernel (inspector, block inspector, executor, census),
    built from the fused integer instructions the design relies on."""
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-sass", build.build()]).decode()
    sections = out.split("Function : ")
    names = [sec.split("\n", 1)[0] for sec in sections[1:]]
    for k in ("k_inspectILi4EE", "k_inspect_nILi4EE", "k_inspect_blockILi4E", "k_executeILi4E", "k_censusILi4E",
              "k_traceback", "k_pack", "k_bin_count", "k_combine_write"):
        assert any(k in n for n in names), k
    insp = next(sec for sec in sections[1:] if sec.startswith("_ZN2fz9k_inspectILi4EE"))
    for mnem in ("VIADDMNMX", "VIMNMX3", "LDS.64", "SHFL.IDX", "VOTE", "IMAD"):
        assert mnem in insp, mnem
