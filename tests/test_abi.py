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
    from paper_conf_icpp_lantra0m24_b200 import build
    lib_path = build.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib_path],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


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
