"""The C ABI library loads and exports every symbol include/ffm.h declares; host-only
calls work without a GPU; compute calls fail loudly without one (no CPU fallback)."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_sc_weltonm19_b200 as ffm

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "ffm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ffm_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    d = _declared()
    for name in ("ffm_log_create", "ffm_log_append", "ffm_dedup_run"):
        assert name in d


def test_library_exports_every_declared_symbol():
    L = ffm.lib()
    for name in _declared():
        assert hasattr(L, name), name
    assert sorted(ffm.EXPORTS) == _declared()
    out = subprocess.run(["nm", "-D", "--defined-only", ffm._LIB_PATH], capture_output=True, text=True).stdout
    syms = {l.split()[-1] for l in out.splitlines() if l.strip()}
    for name in _declared():
        assert name in syms, name


def test_library_is_sm100a_only():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", ffm._LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "sm_90" not in out and "sm_80" not in out


def test_host_only_calls():
    c = ffm.ffm_config_init()
    assert c.digest_bits == 64 and c.refine_bits == 64 and c.world == 1 and c.n_sites == 1
    assert ffm.ffm_strerror(ffm.FFM_E_RANGE) == "argument out of range"
    assert "sm_100a" in ffm.ffm_version()
    assert ffm.lib().ffm_log_destroy(None) == 0
    assert ffm.ffm_log_count(None) == 0


def test_bad_config_rejected_before_device():
    c = ffm.ffm_config_init()
    c.n_sites = 0
    with pytest.raises(ffm.FfmError) as e:
        ffm.ffm_log_create(c)
    assert e.value.code == ffm.FFM_E_INVAL
    c = ffm.ffm_config_init()
    c.chunk_bytes = 1000
    with pytest.raises(ffm.FfmError) as e:
        ffm.ffm_log_create(c)
    assert e.value.code == ffm.FFM_E_INVAL


@pytest.mark.skipif(os.path.exists("/dev/nvidia0"), reason="a GPU is present")
def test_no_cpu_fallback_without_gpu():
    c = ffm.ffm_config_init()
    with pytest.raises(ffm.FfmError) as e:
        ffm.ffm_log_create(c)
    assert e.value.code == ffm.FFM_E_NODEV


def test_product_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_weltonm19_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cpp", ".cuh")):
                txt = open(os.path.join(dirpath, f)).read()
                for bad in ("import oracle", "from oracle", "ffm_oracle", "loggen"):
                    assert bad not in txt, (f, bad)
    out = subprocess.run(["nm", "-D", ffm._LIB_PATH], capture_output=True, text=True).stdout
    assert "oracle" not in out


def test_binding_constants_match_the_header():
    """Every FFM_* enum value include/ffm.h defines has the same value in the binding."""
    src = re.sub(r"/\*.*?\*/", "", open(os.path.join(ROOT, "include", "ffm.h")).read(), flags=re.S)
    consts = {m.group(1): int(m.group(2)) for m in re.finditer(r"\b(FFM_[A-Z_0-9]+)\s*=\s*(-?\d+)u?\b", src)}
    assert {"FFM_OK", "FFM_E_NODEV", "FFM_PAYLOAD_DEVICE", "FFM_FLAG_ONLINE", "FFM_FLAG_APPEND_HASH",
            "FFM_SHARD_CONTIGUOUS"} <= set(consts)
    for name, value in consts.items():
        assert getattr(ffm, name) == value, name
