"""The Python binding's ctypes mirrors of the C-ABI structs (sched.py) have
the size and field offsets of include/sched.h as compiled by the C compiler
(a tiny gcc program prints sizeof / offsetof): a field added on one side only
would shift every later field silently."""
import ctypes as C
import os
import subprocess
import tempfile

import pytest

from paper_conf_sc_weaverkmeh0m24_b200 import sched as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

MIRRORS = {"sched_profile": B._Profile, "sched_query": B._Query, "sched_pick": B.Pick,
           "sched_stats": B.Stats, "sched_dp_point": B.DPPoint, "sched_split_pick": B.SplitPick}


def _c_layout():
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "sched.h"', 'int main(void) {']
    for cname, py in MIRRORS.items():
        lines.append(f'  printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'  printf("{cname} {f} %zu\\n", offsetof({cname}, {f}));')
    lines.append('  return 0;\n}')
    with tempfile.TemporaryDirectory() as d:
        src, exe = os.path.join(d, "abi.c"), os.path.join(d, "abi")
        open(src, "w").write("\n".join(lines))
        r = subprocess.run(["gcc", "-std=c11", "-iquote", os.path.join(ROOT, "include"), "-o", exe, src],
                           capture_output=True, text=True)
        if r.returncode != 0:
            pytest.fail(r.stderr[-2000:])
        out = subprocess.run([exe], capture_output=True, text=True, check=True).stdout
    lay = {}
    for line in out.splitlines():
        name, field, val = line.split()
        lay[(name, field)] = int(val)
    return lay


def test_ctypes_mirrors_match_the_header():
    lay = _c_layout()
    for cname, py in MIRRORS.items():
        assert C.sizeof(py) == lay[(cname, "size")], cname
        for f, _ in py._fields_:
            assert getattr(py, f).offset == lay[(cname, f)], (cname, f)
