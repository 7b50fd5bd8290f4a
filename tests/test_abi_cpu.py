"""C-ABI library checks that need no GPU: it loads, exports every symbol include/lmatch.h declares,
the ctypes mirrors match the header's structs, and argument errors that are decided on the host
return the documented status codes without touching CUDA."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "lmatch.h")


@pytest.fixture(scope="module")
def pkg():
    lib = os.path.join(ROOT, "paper_conf_sc_mandulakgfhs24_b200", "liblmatch.so")
    if not os.path.exists(lib):
        subprocess.check_call(["make", "-C", ROOT, "paper_conf_sc_mandulakgfhs24_b200/liblmatch.so"])
    import paper_conf_sc_mandulakgfhs24_b200 as p
    return p


def declared_functions():
    src = open(HEADER).read()
    return re.findall(r"LMATCH_API\s+[\w\s\*]+?\b(lmatch_\w+)\s*\(", src)


def test_header_declares_api():
    names = declared_functions()
    for must in ("lmatch_create", "lmatch_run", "lmatch_weight", "lmatch_destroy"):
        assert must in names


def test_exports_every_declared_symbol(pkg):
    out = subprocess.check_output(["nm", "-D", "--defined-only", pkg.lib_path]).decode()
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    missing = [f for f in declared_functions() if f not in exported]
    assert not missing, missing
    # nothing else leaks: only lmatch_* symbols are exported as functions
    extra = [s for s in exported if not s.startswith("lmatch_")]
    assert not extra, extra[:10]


def test_links_no_torch_and_static_cudart(pkg):
    out = subprocess.check_output(["ldd", pkg.lib_path]).decode()
    assert "torch" not in out and "libcudart.so" not in out


def test_struct_layout_matches_header(pkg):
    # compile a tiny C program against the header and compare sizeof/offsetof
    src = r'''
#include <stdio.h>
#include <stddef.h>
#include "lmatch.h"
int main(void){
  printf("%zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu\n", sizeof(lmatch_opts), sizeof(lmatch_stats),
         offsetof(lmatch_stats, weight), offsetof(lmatch_stats, ms_sweep),
         offsetof(lmatch_opts, upload_chunk), offsetof(lmatch_opts, host_cache),
         offsetof(lmatch_opts, batches), offsetof(lmatch_stats, cache_rows),
         offsetof(lmatch_stats, cache_bytes), offsetof(lmatch_opts, algorithm),
         offsetof(lmatch_stats, tail_passes), offsetof(lmatch_opts, sort_chunk_log2));
  return 0; }'''
    tmp = os.path.join(ROOT, "build")
    os.makedirs(tmp, exist_ok=True)
    c = os.path.join(tmp, "layout.c")
    exe = os.path.join(tmp, "layout")
    open(c, "w").write(src)
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
    got = [int(x) for x in subprocess.check_output([exe]).split()]
    S, O = pkg.Stats, pkg.Opts
    assert got == [ctypes.sizeof(O), ctypes.sizeof(S), S.weight.offset, S.ms_sweep.offset,
                   O.upload_chunk.offset, O.host_cache.offset, O.batches.offset,
                   S.cache_rows.offset, S.cache_bytes.offset, O.algorithm.offset,
                   S.tail_passes.offset, O.sort_chunk_log2.offset]


def test_host_side_argument_errors(pkg):
    off = np.zeros(2, np.int64)
    col = np.zeros(0, np.int32)
    w = np.zeros(0, np.float32)
    h = ctypes.c_void_p()
    lib = pkg._lib
    assert lib.lmatch_create(off.ctypes.data, col.ctypes.data, w.ctypes.data, -1, 0,
                             ctypes.byref(h)) == pkg.LMATCH_ERANGE
    assert lib.lmatch_create(off.ctypes.data, col.ctypes.data, w.ctypes.data, 1 << 31, 0,
                             ctypes.byref(h)) == pkg.LMATCH_ERANGE
    assert lib.lmatch_create(None, None, None, 1, 0, ctypes.byref(h)) == pkg.LMATCH_EINVAL
    assert lib.lmatch_create(off.ctypes.data, None, None, 1, 4, ctypes.byref(h)) == pkg.LMATCH_EINVAL
    assert lib.lmatch_create(off.ctypes.data, col.ctypes.data, w.ctypes.data, 1, 0,
                             None) == pkg.LMATCH_EINVAL
    assert h.value is None
    assert lib.lmatch_run(None, None, None) == pkg.LMATCH_ESTATE
    assert lib.lmatch_info(None, None, None, None, None) == pkg.LMATCH_ESTATE
    lib.lmatch_destroy(None)  # NULL-safe
    assert pkg.lmatch_strerror(pkg.LMATCH_EINVAL).startswith("invalid")
    assert pkg.lmatch_abi_version() == 4
    assert pkg.lmatch_strerror(pkg.LMATCH_EROUNDS).startswith("round cap")
    assert "n" in pkg.lmatch_last_error() or pkg.lmatch_last_error() == ""


def test_no_oracle_in_product():
    """The product package never imports/links the oracle (test infrastructure only)."""
    pdir = os.path.join(ROOT, "paper_conf_sc_mandulakgfhs24_b200")
    for dirpath, _, files in os.walk(pdir):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in txt.lower().replace("oracle_free", ""), f
