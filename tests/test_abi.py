"""CPU-side checks of the C-ABI boundary: the library builds and loads, it
exports every symbol include/abs.h declares, the ctypes mirrors of the ABI
structs have the C layout, and without an sm_100 GPU the library fails
loudly (no CPU fallback).  No compute calls."""
from __future__ import annotations

import ctypes as C
import os
import re
import subprocess

import pytest

import paper_conf_icpp_yasudonitkyi20_b200 as abs_b200
from paper_conf_icpp_yasudonitkyi20_b200 import abs as binding

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "abs.h")


def declared_symbols():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^ABS_API\s+[\w\s\*]*?\b(abs_\w+)\s*\(", txt, flags=re.M)))


def test_library_exports_every_declared_symbol():
    lib = abs_b200.load()
    names = declared_symbols()
    assert len(names) >= 15
    out = subprocess.check_output(["nm", "-D", "--defined-only", abs_b200.library_path()]).decode()
    exported = set(re.findall(r"\bT (abs_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    for n in names:
        assert hasattr(lib, n)
    assert set(binding.EXPORTS) == set(names)


def test_sm100a_only_cubin():
    out = subprocess.check_output(["cuobjdump", "--list-elf", abs_b200.library_path()]).decode()
    assert "sm_100a" in out
    sass = subprocess.check_output(["cuobjdump", "-sass", abs_b200.library_path()]).decode()
    assert "UBLKCP" in sass            # TMA bulk copy of W rows (cp.async.bulk)
    assert "REDUX" in sass             # warp argmin via redux.sync


def test_struct_layout_matches_c(tmp_path):
    src = tmp_path / "lay.c"
    src.write_text(r'''
#include <stdio.h>
#include <stddef.h>
#include "abs.h"
int main(void){
  printf("%zu %zu %zu %zu %zu %zu\n", sizeof(abs_config), offsetof(abs_config, seed),
         offsetof(abs_config, mode), sizeof(abs_stats), offsetof(abs_stats, search_seconds),
         offsetof(abs_stats, kernel_launches));
  return 0; }
''')
    exe = tmp_path / "lay"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    vals = [int(v) for v in subprocess.check_output([str(exe)]).split()]
    assert vals == [C.sizeof(binding.abs_config), binding.abs_config.seed.offset, binding.abs_config.mode.offset,
                    C.sizeof(binding.abs_stats), binding.abs_stats.search_seconds.offset,
                    binding.abs_stats.kernel_launches.offset]


def test_config_defaults():
    cfg = binding.abs_config()
    abs_b200.load().abs_config_init(C.byref(cfg))
    assert cfg.searches == 0 and cfg.seed == 1 and cfg.mode == binding.MODE_LOCKSTEP and cfg.device == -1
    assert cfg.p_cross == -1 and cfg.p_mut == -1


def test_strerror_and_version():
    L = abs_b200.load()
    assert L.abs_strerror(0) == b"ok"
    assert L.abs_strerror(binding.ABS_EINVAL) == b"invalid argument"
    assert b"sm_100a" in L.abs_version()


def test_fails_loudly_without_gpu():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import numpy as np
    with pytest.raises(abs_b200.AbsError) as e:
        abs_b200.Solver(np.zeros((8, 8), np.int16), searches=1)
    assert e.value.rc == binding.ABS_ECUDA


def test_null_arguments_rejected():
    L = abs_b200.load()
    assert L.abs_create(None, 8, None, None) == binding.ABS_EINVAL
    assert L.abs_search(None, 1) == binding.ABS_EINVAL
    assert L.abs_best(None, None, None) == binding.ABS_EINVAL
