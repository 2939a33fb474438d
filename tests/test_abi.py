"""Host-side checks of the C-ABI boundary (no GPU needed, no compute calls).

* libboids.so builds for sm_100a and exports every function include/boids.h declares;
* the header's structs have the layout the ctypes binding assumes (checked by
  compiling a probe against the header with gcc);
* argument validation returns BOIDS_EINVAL before touching the device;
* the product package never imports the oracle, and the two share no source.
"""
import ctypes as C
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "boids.h")
PKG = os.path.join(ROOT, "paper_conf_ipps_breitbart09_b200")


def header_functions():
    txt = open(HDR).read()
    return sorted(set(re.findall(r"BOIDS_API\s+[\w\s\*]+?\b(boids_\w+)\s*\(", txt)))


def test_header_declares_exports():
    from paper_conf_ipps_breitbart09_b200 import abi

    assert header_functions() == sorted(abi.EXPORTS)


def test_library_exports_every_symbol(boidslib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", boidslib._name], text=True)
    syms = {l.split()[-1] for l in out.splitlines() if l.strip()}
    missing = [f for f in header_functions() if f not in syms]
    assert not missing, missing
    for f in header_functions():
        getattr(boidslib, f)


def test_sass_is_sm100a(boidslib):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", boidslib._name], text=True)
    assert "sm_100a" in out


def test_struct_layout_matches_header(tmp_path):
    from paper_conf_ipps_breitbart09_b200 import abi

    src = tmp_path / "probe.c"
    src.write_text('#include <stddef.h>\n#include <stdio.h>\n#include "boids.h"\n'
                   'int main(void){printf("%zu %zu %zu %zu %zu %zu %zu\\n", sizeof(boids_params), '
                   'offsetof(boids_params, think_every), sizeof(boids_info_t), '
                   'offsetof(boids_info_t, cluster), offsetof(boids_info_t, step_index), '
                   'offsetof(boids_info_t, last_path), offsetof(boids_info_t, steps_sorted));return 0;}\n')
    exe = tmp_path / "probe"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = list(map(int, subprocess.check_output([str(exe)], text=True).split()))
    assert got == [C.sizeof(abi.boids_params), abi.boids_params.think_every.offset,
                   C.sizeof(abi.boids_info_t), abi.boids_info_t.cluster.offset,
                   abi.boids_info_t.step_index.offset, abi.boids_info_t.last_path.offset,
                   abi.boids_info_t.steps_sorted.offset]


def test_default_params_match_design_table(boidslib, orc):
    from paper_conf_ipps_breitbart09_b200 import abi

    p = abi.boids_default_params()
    o = orc.default_params()
    for name, _ in abi.boids_params._fields_:
        assert getattr(p, name) == getattr(o, name), name
    assert p.max_neighbors == 7


@pytest.mark.parametrize("field,value", [("max_neighbors", 8), ("search_radius", 0.0),
                                         ("search_radius", float("nan")), ("mass", 0.0),
                                         ("search_mode", 5), ("init_mode", -1), ("max_speed", -1.0),
                                         ("think_every", 0)])
def test_create_rejects_bad_params(boidslib, field, value):
    from paper_conf_ipps_breitbart09_b200 import abi

    p = abi.boids_default_params(**{field: value})
    with pytest.raises(abi.BoidsError) as e:
        abi.boids_create(100, p, 1)
    assert e.value.code == abi.BOIDS_EINVAL


def test_create_rejects_bad_sizes(boidslib):
    from paper_conf_ipps_breitbart09_b200 import abi

    for n in (0, -5):
        with pytest.raises(abi.BoidsError) as e:
            abi.boids_create(n, None, 1)
        assert e.value.code == abi.BOIDS_EINVAL
    with pytest.raises(abi.BoidsError) as e:
        abi.boids_create_shard(100, None, 1, 3, 2)
    assert e.value.code == abi.BOIDS_EINVAL


def test_null_handle_calls_fail_cleanly(boidslib):
    assert boidslib.boids_step(None, C.c_float(0.1), 1) == -1
    assert boidslib.boids_sync(None) == -1
    assert boidslib.boids_get_state(None, None, None, None, None, None) == -1
    boidslib.boids_destroy(None)  # no-op


def test_product_never_imports_oracle():
    for dp, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", txt, re.M), f
                assert "boids_oracle" not in txt and "liboracle" not in txt, f


def test_oracle_and_cuda_share_no_source():
    orc_src = open(os.path.join(ROOT, "oracle", "boids_oracle.c")).read()
    incs = re.findall(r'#include\s+[<"]([^>"]+)[>"]', orc_src)
    assert all(i in ("math.h", "stdint.h", "stdlib.h", "string.h") for i in incs), incs


def test_partition_rule():
    from paper_conf_ipps_breitbart09_b200.shard import partition

    for n in (1, 7, 1000, 131072, 1048576, 1000003):
        for world in (1, 2, 3, 4, 8):
            spans = [partition(n, world, r) for r in range(world)]
            m = spans[0][2]
            assert m % 256 == 0 and m * world >= n
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (lo, hi, mm), (lo2, _, _) in zip(spans, spans[1:]):
                assert hi == lo2 and mm == m and hi - lo <= m
