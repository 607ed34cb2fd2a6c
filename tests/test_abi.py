"""C-ABI library checks that need no GPU: the in-tree .so builds/loads, exports every symbol
include/wjindex.h declares, and fails loudly (WJ_ERR_CUDA) when no CUDA device is present."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_ipps_weij11_b200 as wj

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "wjindex.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(index_\w+)\s*\(", src)))


def test_header_declares_the_binding_names():
    assert declared_functions() == sorted(wj.EXPORTS)


def test_library_exports_every_declared_symbol():
    lib = wj.load_library()
    for name in declared_functions():
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", wj.LIB_PATH], capture_output=True, text=True).stdout
    for name in declared_functions():
        assert re.search(rf"\bT {name}$", out, re.M), name


def test_library_is_sm100a():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", wj.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_struct_sizes_match_header(tmp_path):
    # wj_config: 3 x i32 + pad + 2 pointers + u64 + 2 x u32 + pointer + u64 = 64 bytes on LP64
    assert ctypes.sizeof(wj.Config) == 64
    # the binding's structs against the C compiler's view of include/wjindex.h
    src = tmp_path / "sz.c"
    src.write_text('#include <stdio.h>\n#include "wjindex.h"\n'
                   'int main(void){printf("%zu %zu %d %d\\n", sizeof(wj_config), sizeof(wj_stats),'
                   ' (int)WJ_PHASE_COUNT, (int)WJ_KERNEL_COUNT); return 0;}\n')
    exe = tmp_path / "sz"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    cfg, sts, nph, nk = map(int, subprocess.run([str(exe)], check=True, capture_output=True, text=True).stdout.split())
    assert ctypes.sizeof(wj.Config) == cfg
    assert ctypes.sizeof(wj.Stats) == sts
    assert len(wj.KERNELS) == nk and nph == 16
    assert wj.NODE_DTYPE.itemsize == 512  # Table II


def test_no_cpu_fallback_without_gpu():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(wj.WJError) as e:
        wj.Index(device=0)
    assert e.value.code == -3  # WJ_ERR_CUDA


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_weij11_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f), errors="ignore").read()
                assert "import oracle" not in txt and "oracle/" not in txt and "oracle.h" not in txt, f


def test_library_stop_list_is_sklearn_english():
    # the CUDA path's own copy of the stop list (reading S20), pinned independently of the oracle's
    text = pytest.importorskip("sklearn.feature_extraction.text")
    words = wj.stop_words()
    assert len(words) == len(set(words)) == 318
    assert sorted(words) == sorted(text.ENGLISH_STOP_WORDS)


def test_debug_stem_validates_without_gpu():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(wj.WJError) as e:
        wj.debug_stem([b"cats"])
    assert e.value.code == -3  # WJ_ERR_CUDA: no CPU fallback
