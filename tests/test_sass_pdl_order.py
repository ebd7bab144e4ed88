"""SASS check of the programmatic-dependent-launch ordering (no GPU needed).

A plain fused kernel is launched with programmatic stream serialisation: its
CTAs start while the preceding kernel still runs and block in
griddepcontrol.wait (SASS ACQBULK) before touching user data.  ptxas may
schedule an ld.global.nc load above that wait (observed on
tools/cfg1_lab.cu: LDG.E.CONSTANT before ACQBULK), so the library's loads that
follow the wait are coherent ones (fused_kernel.cu kNcLoads).  This test
disassembles libddt.so and checks, for every parameter-batch instance of the
closed-form variants (no commit-time list tables that may legally be read
before the wait), that no global load precedes the first ACQBULK and that no
load at all takes the non-coherent path.
"""
import os
import re
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_cluster_chukzsp20_b200", "libddt.so")
CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"


def _functions():
    if not os.path.exists(LIB) or not os.path.exists(CUOBJDUMP):
        pytest.skip("libddt.so or cuobjdump missing")
    txt = subprocess.run([CUOBJDUMP, "-sass", LIB], capture_output=True, text=True, check=True).stdout
    out = {}
    for f in re.split(r"\n\s*Function : ", txt)[1:]:
        name = f.split("\n", 1)[0].strip()
        out[name] = [m.group(1) for m in re.finditer(r"/\*[0-9a-f]{4}\*/\s+(.*?);", f)]
    return out


def test_no_data_load_before_the_pdl_wait():
    funcs = _functions()
    checked = 0
    for name, ins in funcs.items():
        m = re.match(r"_ZN3ddt15ddt_fused_paramILi(\d+)ELi(\d+)E", name)
        if not m or int(m.group(2)) not in (1, 2, 3, 4, 5, 7, 9):
            continue
        acq = [i for i, x in enumerate(ins) if x.startswith("ACQBULK")]
        assert acq, f"{name}: no griddepcontrol.wait"
        early = [x for x in ins[:acq[0]] if re.match(r"(@!?U?P\d+\s+)?LDG", x)]
        assert not early, f"{name}: global loads before the PDL wait: {early[:3]}"
        # the closed-form variants read no commit-time list table, so no load of theirs may take the
        # non-coherent path (LDG ... CONSTANT) that ptxas is free to move above the wait
        nc = [x for x in ins if re.match(r"(@!?U?P\d+\s+)?LDG\S*CONSTANT", x)]
        assert not nc, f"{name}: non-coherent loads in a PDL kernel: {nc[:3]}"
        checked += 1
    assert checked >= 14, checked  # 7 variants x 2 parameter forms
