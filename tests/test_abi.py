"""The C-ABI library loads and exports every symbol include/song.h declares
(CPU only: no compute call is made without a GPU)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "song.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(song_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_boundary():
    names = declared_functions()
    for required in ("song_index_create", "song_search", "song_index_destroy"):
        assert required in names
    assert len(names) >= 10


def test_library_exports_every_declared_symbol():
    from paper_conf_icde_zhaotl20_b200 import song
    lib = song.lib()
    for name in declared_functions():
        assert hasattr(lib, name), name
    assert sorted(song.EXPORTED) == declared_functions()
    assert song.version().startswith("song-b200")
    assert "sm_100a" in song.version()


def test_library_is_built_for_sm100a():
    from paper_conf_icde_zhaotl20_b200 import song
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", song.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_argument_errors_need_no_gpu():
    """Argument validation happens before any CUDA call."""
    from paper_conf_icde_zhaotl20_b200 import song
    lib = song.lib()
    out = ctypes.c_void_p()
    rc = lib.song_index_create(None, 10, 4, None, 4, 0, ctypes.byref(out))
    assert rc == -1 and b"NULL" in lib.song_last_error()
    assert lib.song_index_destroy(None) == 0
    p = song.SearchParams()
    lib.song_default_params(ctypes.byref(p), 10, 64)
    assert (p.K, p.queue_len, p.visited, p.entry, p.id_offset, p.steps) == (10, 64, 0, 0, 0, 0)
    buf = (ctypes.c_float * 8)()
    rc = lib.song_search_pipelined(None, ctypes.byref(p), buf, 1, 1, buf, buf)
    assert rc == -1 and b"NULL" in lib.song_last_error()


def test_union_is_the_default_queue():
    """Reading R17 (one bounded list W of q and topk) is what the library runs
    by default with the hash visited set and one pop per iteration: in
    registers up to queue_len 256, in shared-memory tiers above; the paper's
    separate q / topk on request, and for the other visited kinds."""
    from paper_conf_icde_zhaotl20_b200 import song
    for L, regs in ((16, 1), (33, 2), (100, 4), (128, 4), (160, 8), (256, 8), (257, 0), (1280, 0)):
        pl = song.plan(song.Params(K=10, queue_len=L), 128)
        assert (pl.queue_kind, pl.queue_regs) == (2, regs), L
    sep = song.plan(song.Params(K=10, queue_len=64, queue_kind="separate"), 128)
    assert (sep.queue_kind, sep.queue_regs) == (0, 2)
    bl = song.plan(song.Params(K=10, queue_len=64, visited="bloom"), 128)
    assert bl.queue_kind == 0
    ms = song.plan(song.Params(K=10, queue_len=64, steps=2), 128)
    assert ms.queue_kind == 0


def test_params_struct_layout_matches_header(tmp_path):
    """The ctypes mirrors have the C compiler's sizes and field offsets."""
    import subprocess
    from paper_conf_icde_zhaotl20_b200 import song
    src = tmp_path / "layout.c"
    src.write_text(
        '#include <stdio.h>\n#include <stddef.h>\n#include "song.h"\n'
        'int main(void){printf("%zu %zu %zu %zu %zu\\n", sizeof(song_search_params),'
        ' sizeof(song_index_info), offsetof(song_index_info, vector_bytes),'
        ' offsetof(song_index_info, code_bits), offsetof(song_search_params, table_log2));'
        'printf("%zu %zu\\n", sizeof(song_search_plan), offsetof(song_search_plan, warps_per_block));'
        'return 0;}\n')
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(src),
                           "-o", str(exe)])
    c = [int(x) for x in subprocess.check_output([str(exe)], text=True).split()]
    assert c == [ctypes.sizeof(song.SearchParams), ctypes.sizeof(song.IndexInfo),
                 song.IndexInfo.vector_bytes.offset, song.IndexInfo.code_bits.offset,
                 song.SearchParams.table_log2.offset, ctypes.sizeof(song.SearchPlan),
                 song.SearchPlan.warps_per_block.offset]


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_zhaotl20_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "song_oracle" not in text and "liboracle" not in text, f


def test_rp_argument_errors_need_no_gpu():
    """§VII entry points validate before any CUDA call."""
    import numpy as np
    from paper_conf_icde_zhaotl20_b200 import song
    lib = song.lib()
    out = ctypes.c_void_p()
    codes = np.zeros((4, 2), np.uint32)
    adj = np.zeros((4, 2), np.int32)
    P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
    assert lib.song_rp_encode(None, 4, 8, None, 64, None, None) == -1
    # bits must be a positive multiple of 32, at most SONG_MAX_CODE_BITS
    assert lib.song_index_create_codes(P(codes), 4, 48, P(adj), 2, ctypes.byref(out)) == -1
    assert lib.song_index_create_codes(P(codes), 4, 0, P(adj), 2, ctypes.byref(out)) == -1
    assert lib.song_index_create_codes(P(codes), 4, 2048, P(adj), 2, ctypes.byref(out)) == -4
    assert lib.song_index_create_codes(None, 4, 64, P(adj), 2, ctypes.byref(out)) == -1
    bad = adj.copy()
    bad[1, 1] = 4  # id out of range
    assert lib.song_index_create_codes(P(codes), 4, 64, P(bad), 2, ctypes.byref(out)) == -1
    assert not out.value
    # float creators reject SONG_HAMMING
    v = np.zeros((4, 8), np.float32)
    assert lib.song_index_create(P(v), 4, 8, P(adj), 2, 3, ctypes.byref(out)) == -1
    R = np.zeros((64, 8), np.float32)
    R[0, 0] = np.nan
    assert lib.song_index_create_rp(P(v), 4, 8, P(R), 64, P(adj), 2, ctypes.byref(out)) == -1


@pytest.mark.parametrize("L", [1, 10, 28, 32, 48, 64, 100, 128, 144, 512, 1280, 2048])
def test_plan_lazy_capacity_bounds(L):
    """song_search_plan_get (host-only) resolves the lazy-deletion capacity C
    of reading R14 inside its stated bounds: C >= 2L + 32 (the live bound
    |q| + |topk| + one iteration's candidates) and C <= 3/4 of the table."""
    from paper_conf_icde_zhaotl20_b200 import song
    p = song.plan(song.Params(K=1, queue_len=L), 128)
    slots = 1 << p.visited_log2
    assert 2 * L + 32 <= p.visited_cap <= 3 * slots // 4
    assert p.queue_regs == (1 if L <= 32 else 2 if L <= 64 else 4 if L <= 128 else 8 if L <= 256 else 0)
    assert p.smem_per_warp * p.warps_per_block <= 227 * 1024
    # eager deletion and multi-step probing report -1; other kinds 0
    assert song.plan(song.Params(K=1, queue_len=L, visited_cap=-1), 128).visited_cap == -1
    assert song.plan(song.Params(K=1, queue_len=L, steps=2), 128).visited_cap == -1
    assert song.plan(song.Params(K=1, queue_len=L, visited="bloom"), 128).visited_cap == 0


def test_plan_errors_need_no_gpu():
    from paper_conf_icde_zhaotl20_b200 import song
    with pytest.raises(song.SongError) as e:  # K > queue_len
        song.plan(song.Params(K=20, queue_len=10), 128)
    assert e.value.code == -1
    with pytest.raises(song.SongError) as e:  # a global table that one iteration could fill
        song.plan(song.Params(K=1, queue_len=10, visited="hashtable", table_log2=6), 128)
    assert e.value.code == -4
    song.plan(song.Params(K=1, queue_len=10, visited="hashtable", table_log2=7), 128)
    with pytest.raises(song.SongError):  # Cuckoo on codes
        song.plan(song.Params(K=1, queue_len=10, visited="cuckoo"), 4, "hamming")
    with pytest.raises(song.SongError):
        song.plan(song.Params(K=1, queue_len=10), 2048)


def _build_c_example(tmp_path):
    import subprocess
    from paper_conf_icde_zhaotl20_b200 import song
    libdir = os.path.dirname(song.LIB_PATH)
    exe = str(tmp_path / "search_example")
    cmd = ["gcc", "-O2", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
           os.path.join(ROOT, "examples", "search_example.c"), "-L", libdir, "-lsong",
           f"-Wl,-rpath,{libdir}", "-lm", "-o", exe]
    res = subprocess.run(cmd, capture_output=True, text=True)
    assert res.returncode == 0, res.stderr
    return exe


def test_c_example_builds_against_the_header(tmp_path):
    """A plain C program (no Python, no torch) compiles against include/song.h
    and links libsong.so; tests/test_gpu_c_example.py runs it on a GPU."""
    assert os.path.exists(_build_c_example(tmp_path))
