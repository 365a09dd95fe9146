"""The C-ABI library loads and exports every entry point include/fleche.h declares (no GPU)."""
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "fleche.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fleche_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    d = _declared()
    for name in ["fleche_create", "fleche_query", "fleche_stats", "fleche_destroy"]:
        assert name in d


def test_library_exports_every_declared_symbol():
    import paper_conf_eurosys_xiellwgrs22_b200 as pkg
    from paper_conf_eurosys_xiellwgrs22_b200 import binding
    nm = subprocess.check_output(["nm", "-D", "--defined-only", pkg.LIB_PATH]).decode()
    exported = set(re.findall(r" T (fleche_\w+)", nm))
    assert set(_declared()) <= exported, set(_declared()) - exported
    assert set(_declared()) == set(binding.EXPORTED)
    assert binding.fleche_strerror(-5).decode().startswith("an ID outside")


def test_kernels_are_sm100a():
    import paper_conf_eurosys_xiellwgrs22_b200 as pkg
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", pkg.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_create_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        return
    import numpy as np
    from paper_conf_eurosys_xiellwgrs22_b200 import FlatCache, FlecheError
    t = np.zeros((10, 4), np.float32)
    try:
        FlatCache([10], [4], [t], 64, 16)
    except FlecheError as e:
        assert e.status in (-1, -3)
    else:
        raise AssertionError("create succeeded without a GPU")
