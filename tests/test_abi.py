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


def test_library_encoder_matches_oracle_on_every_config():
    """fleche_encode (the code fleche_create builds; host-only, no GPU) against the oracle's
    independently written encoder (reading R3) for every BASELINE config,
    including cfg3's 31-bit Terabyte code, and the short-key fallback (reading R24)."""
    import numpy as np
    from oracle import oracle as O
    from paper_conf_eurosys_xiellwgrs22_b200 import binding
    from workload import configs
    for name in ("cfg0", "cfg1", "cfg2", "cfg3", "cfg3h", "cfg4", "cfg5"):
        w = configs.get(name)
        kb, base, fb, h = binding.encode(w.cards)
        bmin, obase, ofb = O.encode(w.cards)
        assert kb == bmin and np.array_equal(base, obase) and np.array_equal(fb, ofb), name
        assert not h.any()
    w = configs.get("cfg2")
    for B in (20, 23, 25):
        kb, base, fb, h = binding.encode(w.cards, B)
        lossy, obase, obits, oex = O.encode_short(w.cards, B)
        assert kb == B and np.array_equal(base, obase) and np.array_equal(fb, obits), B
        assert np.array_equal(h, 1 - oex) and int(h.sum()) == lossy
    try:
        binding.encode([1 << 31] * 4)  # 33-bit exact code: rejected
    except binding.FlecheError as e:
        assert e.status == binding.EINVAL
    else:
        raise AssertionError("a code wider than 32 bits was accepted")


def test_binding_rejects_bad_buffers():
    """The binding validates dtype / contiguity / device / size before any pointer reaches
    the C ABI (an int32 or host ID array, or a short out buffer, would otherwise make the
    kernels read or write out of bounds)."""
    import numpy as np
    import pytest
    import torch
    from paper_conf_eurosys_xiellwgrs22_b200.binding import _check_ids, _check_out
    with pytest.raises(ValueError):
        _check_ids([np.zeros(4, np.int32)], 1, None, "q")
    with pytest.raises(ValueError):
        _check_ids([np.zeros(4, np.int64)], 2, None, "q")  # wrong table count
    with pytest.raises(ValueError):
        _check_ids([torch.zeros(4, dtype=torch.int64)], 1, 0, "q")  # host tensor for the device path
    with pytest.raises(ValueError):
        _check_ids([torch.zeros(8, dtype=torch.int64)[::2]], 1, None, "q")  # not contiguous
    _check_ids([np.zeros(4, np.int64), 1234], 2, None, "q")  # raw pointers pass through
    with pytest.raises(ValueError):
        _check_out(np.zeros(10, np.float32), 11, None, "q")
    with pytest.raises(ValueError):
        _check_out(np.zeros(16, np.float64), 11, None, "q")
    with pytest.raises(ValueError):
        _check_out(torch.zeros(16), 11, 0, "q")  # host tensor for the device path
    _check_out(np.zeros(11, np.float32), 11, None, "q")
