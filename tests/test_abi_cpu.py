"""CPU-side checks of the C ABI: libbted.so loads, exports every function
include/bted.h declares, and fails loudly (no CPU fallback) without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from paper_conf_date_sunbg021_b200.build import LIB, ROOT
from tests.conftest import cuda_available

HEADER = os.path.join(ROOT, "include", "bted.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\*?\s+(bted_[A-Za-z_]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_library_built_for_sm100a():
    assert os.path.exists(LIB), "run __graft_entry__.build() first"
    out = os.popen(f"cuobjdump --list-elf {LIB} 2>&1").read()
    assert "sm_100a" in out


def test_exports_every_declared_symbol():
    names = declared_functions()
    assert len(names) >= 18
    lib = ctypes.CDLL(LIB)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    assert set(names) == set(L.EXPORTS), set(names) ^ set(L.EXPORTS)


def test_status_strings_and_defaults():
    lib = L.lib()
    assert lib.bted_status_string(0) == b"BTED_OK"
    assert lib.bted_status_string(5) == b"BTED_ENUMERIC"
    p = L.default_params()
    assert p.gamma == 1.0 and p.device == -1 and p.num_batches == 1 and p.flags == 0


@pytest.mark.skipif(cuda_available(), reason="checks the no-GPU failure path")
def test_no_gpu_fails_loudly():
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(np.zeros((4, 2), np.float32), 1.0)
    assert e.value.status == 3 and "no CPU fallback" in str(e.value)
    with pytest.raises(bt.BtedError):
        bt.bted_sample_batches(100, 10, 1, 0)


def test_argument_validation_before_device():
    with pytest.raises(bt.BtedError) as e:
        bt.bted_sample_batches(10, 11, 1, 0)
    assert e.value.status == 1
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(np.zeros((4, 65), np.float32), 1.0)      # d > 64
    assert e.value.status == 1
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(np.zeros((4, 2), np.float32), 0.0)       # gamma <= 0
    assert e.value.status == 1


def test_decode_keys_roundtrip():
    score = np.array([0.5, 0.0, 3.25], np.float32)
    idx = np.array([7, 0, 123456], np.int64)
    keys = ((score.view(np.uint32).astype(np.uint64) + np.uint64(1)) << np.uint64(32)) | \
        (np.uint64(0xFFFFFFFF) - idx.astype(np.uint64))
    i2, s2 = L.decode_keys(keys)
    assert np.array_equal(i2, idx) and np.array_equal(s2, score)


def test_product_path_shares_nothing_with_the_oracle():
    """The product package (Python binding + CUDA sources) never imports, links
    or includes anything under oracle/, and the oracle never imports the product
    package: the two meet only through synth/ inputs and the tests."""
    pkg = os.path.join(ROOT, "paper_conf_date_sunbg021_b200")
    bad = []
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                if re.search(r"^\s*(from|import)\s+oracle\b|#include\s+[\"<][^\">]*oracle|ted_oracle", src, flags=re.M):
                    bad.append(f)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            src = open(os.path.join(ROOT, "oracle", f)).read()
            if re.search(r"^\s*(from|import)\s+paper_conf_date_sunbg021_b200\b|#include\s+[\"<][^\">]*"
                         r"(paper_conf_date_sunbg021_b200|bted)|libbted", src, flags=re.M):
                bad.append("oracle/" + f)
    assert not bad, bad


def test_params_struct_layout_matches_header(tmp_path):
    """The ctypes mirror of bted_params has the header's field offsets and size
    (compiled against include/bted.h by gcc)."""
    fields = [f for f, _ in L.bted_params._fields_]
    src = tmp_path / "layout.c"
    src.write_text('#include <stddef.h>\n#include <stdio.h>\n#include "bted.h"\nint main(void){\n'
                   + "".join(f'printf("{f} %zu\\n", offsetof(bted_params, {f}));\n' for f in fields)
                   + 'printf("SIZE %zu\\n", sizeof(bted_params)); return 0; }\n')
    exe = tmp_path / "layout"
    assert os.system(f"gcc -I{os.path.join(ROOT, 'include')} {src} -o {exe}") == 0
    out = dict(line.split() for line in os.popen(str(exe)).read().splitlines())
    for f in fields:
        assert int(out[f]) == getattr(L.bted_params, f).offset, f
    assert int(out["SIZE"]) == ctypes.sizeof(L.bted_params)
    p = L.default_params()
    assert p.num_devices == 1 and p.norm_mode == 0


def test_multi_device_params_validated_before_device():
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(np.zeros((4, 2), np.float32), 1.0, norm_mode=2)
    assert e.value.status == 1
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(np.zeros((4, 2), np.float32), 1.0, num_devices=-1)
    assert e.value.status == 1


def test_update_checks_host_arrays_before_the_call():
    """bted_update's binding: a host array of the wrong shape is rejected in Python,
    before any pointer reaches the library; the accepted array is converted to C-contiguous fp32."""
    with pytest.raises(ValueError):
        L.bted_update(0, np.zeros((5, 3), np.float32), shape=(4, 3))
    with pytest.raises(ValueError):
        L.bted_update(0, np.zeros((12,), np.float32), shape=(4, 3))
    # a null context with a well-formed array reaches the library, which refuses it (EINVAL)
    with pytest.raises(bt.BtedError) as e:
        L.bted_update(0, np.zeros((4, 3), np.float64).T.copy().T, shape=(4, 3))
    assert e.value.status == 1
