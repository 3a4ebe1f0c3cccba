"""The C-ABI library loads and exports every symbol include/gsap.h declares (no GPU needed)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def libgsap():
    from paper_conf_icpp_changzh24_b200 import build
    build.build()
    return ctypes.CDLL(build.LIB)


def declared():
    src = open(os.path.join(ROOT, "include", "gsap.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gsap_[a-z_]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    names = declared()
    for n in ("gsap_partition", "gsap_propose", "gsap_delta_mdl", "gsap_update_blockmodel", "gsap_mdl"):
        assert n in names


def test_every_declared_symbol_is_exported(libgsap):
    for name in declared():
        assert hasattr(libgsap, name), name


def test_binding_covers_every_symbol(libgsap):
    from paper_conf_icpp_changzh24_b200 import gsap
    assert sorted(gsap.EXPORTED) == declared()


def test_default_params_table2(libgsap):
    from paper_conf_icpp_changzh24_b200 import gsap
    p = gsap.gsap_default_params()
    assert (p.reduction_rate, p.num_proposals, p.max_nodal_itr, p.thresh1, p.thresh2, p.window,
            p.num_batches) == (0.4, 10, 100, 5e-4, 1e-4, 3, 4)        # Table 2
    assert p.beta == 3.0 and p.seed == 0x5B9D2024


def test_struct_layout_matches_header():
    """ctypes mirrors of the header structs: field order / sizes (checked with gcc)."""
    import subprocess
    import tempfile
    from paper_conf_icpp_changzh24_b200 import gsap
    prog = r'''
#include <stdio.h>
#include <stddef.h>
#include "gsap.h"
int main(void){printf("%zu %zu %zu %zu %zu %zu %zu %zu %d\n", sizeof(gsap_params), sizeof(gsap_stats),
  sizeof(gsap_dist), offsetof(gsap_stats, k_move_ms), offsetof(gsap_params, profile),
  offsetof(gsap_stats, t_rebuild), offsetof(gsap_stats, t_comm), offsetof(gsap_stats, n_move_eval),
  GSAP_TRACE_COLS);return 0;}
'''
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "t.c")
        open(c, "w").write(prog)
        exe = os.path.join(d, "t")
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        got = list(map(int, subprocess.check_output([exe]).split()))
    want = [ctypes.sizeof(gsap.gsap_params), ctypes.sizeof(gsap.gsap_stats), ctypes.sizeof(gsap.gsap_dist),
            gsap.gsap_stats.k_move_ms.offset, gsap.gsap_params.profile.offset,
            gsap.gsap_stats.t_rebuild.offset, gsap.gsap_stats.t_comm.offset, gsap.gsap_stats.n_move_eval.offset,
            gsap.TRACE_COLS]
    assert got == want


def test_no_gpu_fails_loudly(libgsap):
    """Without a device the product path returns an error; it never falls back to the CPU."""
    import numpy as np
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_icpp_changzh24_b200 import gsap
    with pytest.raises(gsap.GsapError):
        gsap.Context(np.array([0, 1], np.int64), np.array([0], np.int32))


def test_product_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icpp_changzh24_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", txt).lower() or f == "__init__.py", f


def test_bench_and_entry_compile():
    """bench.py / __graft_entry__.py are valid Python (the driver runs them on the GPU box)."""
    import py_compile
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    for f in ("bench.py", "__graft_entry__.py"):
        py_compile.compile(os.path.join(root, f), doraise=True)


def test_bench_reference_arm_json():
    """`bench.py --impl reference` (the oracle arm) prints one JSON line with the
    contract's keys (run on the 1K config so it takes a second)."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--impl", "reference", "--config", "1k",
                          "--steps", "1", "--warmup", "0"], capture_output=True, text=True, timeout=300, cwd=root)
    assert out.returncode == 0, out.stderr
    line = json.loads(out.stdout.strip().splitlines()[-1])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "cpu_baseline", "e2e", "config"):
        assert k in line, k
    assert line["impl"] == "reference" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0
