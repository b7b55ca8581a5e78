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
    assert (p.K, p.queue_len, p.visited, p.entry, p.id_offset) == (10, 64, 0, 0, 0)


def test_params_struct_layout_matches_header():
    from paper_conf_icde_zhaotl20_b200 import song
    assert ctypes.sizeof(song.SearchParams) == 40
    assert ctypes.sizeof(song.IndexInfo) == 48


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_zhaotl20_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "song_oracle" not in text and "liboracle" not in text, f
