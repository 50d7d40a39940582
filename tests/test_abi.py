"""The C-ABI library builds for sm_100a, loads without a GPU, and exports
every symbol include/opp.h declares (no compute calls here)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "opp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(opp_[a-z_0-9]+)\s*\(", src)))


def test_library_builds_and_exports_every_declared_symbol():
    from paper_conf_icpp_lantra0m24_b200 import build
    lib_path = build.build()
    lib = ctypes.CDLL(lib_path)
    declared = _declared()
    assert len(declared) >= 18
    for name in declared:
        assert hasattr(lib, name), name
    from paper_conf_icpp_lantra0m24_b200 import opp
    assert sorted(opp.EXPORTS) == declared


def test_sass_is_sm100a_and_has_no_fp64_fma_in_push():
    """S11: the push and the barycentric coordinates are evaluated without FMA
    contraction, as the oracle (-ffp-contract=off) evaluates them.  Every
    instance of the particle-loop kernels (pass 1 tiled / direct / tail, the
    continuation) must contain fp64 multiplies and adds but no DFMA."""
    from paper_conf_icpp_lantra0m24_b200 import build
    lib_path = build.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib_path],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib_path],
                          capture_output=True, text=True).stdout
    secs = re.split(r"\n\s*Function : ", sass)[1:]
    hot = [sec for sec in secs if any(k in sec.split("\n", 1)[0]
                                      for k in ("k_push_move_deposit", "k_walk_refill"))]
    assert len(hot) >= 40   # 3 deposit modes x 3 DH modes x (1, N ranks) x (tiled, direct, tail) + refill
    for sec in hot:
        name = sec.split("\n", 1)[0].strip()
        assert "DMUL" in sec and "DADD" in sec, name
        assert not re.search(r"\bDFMA\b", sec), f"fp64 FMA in {name}"


def test_defaults_and_errors_without_gpu():
    from paper_conf_icpp_lantra0m24_b200 import opp
    p = opp.opp_init_params_default()
    assert p.nranks == 1 and p.hop_cap == 1024 and p.hop_budget_per_pass == 4
    assert p.deposit_mode == opp.OPP_DEP_ATOMIC
    bad = opp.opp_init_params_default()
    bad.nranks = 0
    with pytest.raises(opp.OppError) as e:
        opp.opp_init(bad)
    assert e.value.code == opp.OPP_ERR_ARG
