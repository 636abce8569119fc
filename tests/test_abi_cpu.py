"""CPU-only checks of the boundary: libsharp.so loads and exports every symbol
that include/sharp.h declares; the binding exposes the same names; the product
package never imports the oracle (task rule 3).  No compute call needs a GPU
here."""
import ast
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icpp_fanjzac15_b200")


def declared_functions():
    src = open(os.path.join(ROOT, "include", "sharp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sharp_[a-z_]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for n in ["sharp_create", "sharp_run", "sharp_run_batch", "sharp_destroy"]:
        assert n in names


def test_library_loads_and_exports_every_declared_symbol():
    lib = ctypes.CDLL(os.path.join(PKG, "libsharp.so"))
    for name in declared_functions():
        assert hasattr(lib, name), name


def test_binding_exposes_same_names():
    import paper_conf_icpp_fanjzac15_b200 as p
    for name in declared_functions():
        assert hasattr(p, name), name


def test_static_strings_without_gpu():
    import paper_conf_icpp_fanjzac15_b200 as p
    assert "sm_100a" in p.sharp_version()
    assert p.sharp_strerror(p.SHARP_EINVAL) == "invalid argument"
    d = p.sharp_default_params()
    assert (d.amount, d.gamma, d.osc_gain, d.osc_scale) == (1.0, 0.5, 0.5, 2.0)


def test_library_is_sm100a_code():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", os.path.join(PKG, "libsharp.so")],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_product_package_never_imports_or_loads_the_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            path = os.path.join(dirpath, f)
            if f.endswith(".py"):
                tree = ast.parse(open(path).read())
                for node in ast.walk(tree):
                    if isinstance(node, ast.Import):
                        assert all(not a.name.startswith("oracle") for a in node.names), path
                    if isinstance(node, ast.ImportFrom):
                        assert not (node.module or "").startswith("oracle"), path
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                assert "liboracle" not in open(path).read(), path
                assert "oracle.h" not in open(path).read(), path


def test_no_cpu_fallback_create_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_icpp_fanjzac15_b200 as p
    with pytest.raises(p.SharpError):
        p.sharp_create()


def test_c_program_links_against_the_abi():
    """tests/c_abi_check.c compiles against include/sharp.h and links
    libsharp.so with plain gcc (no GPU needed to build)."""
    import subprocess
    exe = os.path.join(ROOT, "tests", "c_abi_check")
    subprocess.run(["make", "-C", ROOT, "-s", "tests/c_abi_check"], check=True)
    assert os.path.exists(exe)
    out = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "libsharp.so" in out and "not found" not in out


def test_reading_switch_values_agree_across_header_binding_and_oracle():
    """SHARP_READ_* (include/sharp.h), the binding's constants and the
    oracle's ORACLE_READ_* are defined independently (no shared code); they
    must name the same bits."""
    hdr = open(os.path.join(ROOT, "include", "sharp.h")).read()
    orc = open(os.path.join(ROOT, "oracle", "oracle.h")).read()
    import oracle
    import paper_conf_icpp_fanjzac15_b200 as p
    for name in ["INT_DOWNSCALE", "COLUMN_WINS", "INTERIOR_MEAN", "STRENGTH_EXP", "OSC_CONST", "TRUNCATE"]:
        h = int(re.search(rf"SHARP_READ_{name}\s*=\s*(\d+)", hdr).group(1))
        o = int(re.search(rf"#define ORACLE_READ_{name}\s+(\d+)", orc).group(1))
        assert h == o == getattr(p, f"SHARP_READ_{name}") == getattr(oracle, f"READ_{name}"), name


def test_config_struct_layout_matches_the_header(tmp_path):
    """The binding's SharpConfig mirrors include/sharp.h's sharp_config (the
    multi-device fields num_devices / device_ids / shard included)."""
    import subprocess
    import paper_conf_icpp_fanjzac15_b200 as p
    src = tmp_path / "layout.c"
    src.write_text('#include <stddef.h>\n#include <stdio.h>\n#include "sharp.h"\n'
                   'int main(void){printf("%zu %zu %zu %zu\\n", sizeof(sharp_config), '
                   'offsetof(sharp_config, num_devices), offsetof(sharp_config, device_ids), '
                   'offsetof(sharp_config, shard)); return 0;}\n')
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)], check=True)
    size, o_n, o_ids, o_sh = map(int, subprocess.run([str(exe)], capture_output=True, text=True).stdout.split())
    C = p.binding.SharpConfig
    assert ctypes.sizeof(C) == size
    assert (C.num_devices.offset, C.device_ids.offset, C.shard.offset) == (o_n, o_ids, o_sh)


def test_band_rows_of_the_abi_match_the_python_partition():
    """sharp_band_rows (the C ABI's row-band partition) equals
    bands.band_rows, tiles [0, h) with multiples of 4, and rejects bad requests."""
    import paper_conf_icpp_fanjzac15_b200 as p
    from paper_conf_icpp_fanjzac15_b200.bands import band_rows
    for h in (8, 12, 1080, 2160, 4320, 16384, 1084):
        for G in range(1, 9):
            if h // 4 < G:
                with pytest.raises(p.SharpError):
                    p.sharp_band_rows(h, G, 0)
                continue
            prev = 0
            for g in range(G):
                r = p.sharp_band_rows(h, G, g)
                assert r == band_rows(h, G, g)
                assert r[0] == prev and r[1] > r[0] and r[0] % 4 == 0 and r[1] % 4 == 0
                prev = r[1]
            assert prev == h
    with pytest.raises(p.SharpError):
        p.sharp_band_rows(1080, 2, 2)
