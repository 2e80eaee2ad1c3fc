"""CPU-side checks of the C-ABI boundary (no GPU needed): the library loads, exports every
symbol include/ss.h declares, its host-only params derivation equals the oracle's
independently computed params, and argument errors come back as status codes."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sslib():
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    return ss


def _declared():
    txt = open(os.path.join(ROOT, "include", "ss.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(ss_[a-z_]+)\s*\(", txt)))


def test_header_symbols_exported(sslib):
    names = _declared()
    assert "ss_orb_extract" in names and "ss_match_projection" in names
    lib = sslib.lib()
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(sslib.EXPORTED) == names


@pytest.mark.parametrize("shape,nf,L", [((752, 480), 1000, 8), ((640, 480), 1000, 8), ((1241, 376), 2000, 8),
                                        ((752, 480), 1250, 8), ((320, 240), 150, 4), ((64, 64), 10, 1),
                                        ((2048, 2048), 5000, 8), ((1000, 100), 300, 2)])
def test_params_equal_oracle(sslib, ref, shape, nf, L):
    p = sslib.ss_orb_params_init(shape[0], shape[1], nf, L)
    q = ref.params(shape[0], shape[1], nf, n_levels=L)
    assert C.string_at(C.addressof(p), C.sizeof(p)) == C.string_at(C.addressof(q), C.sizeof(q))


def test_params_reject(sslib):
    for args in ((40, 40, 1000), (752, 480, 0), (752, 480, 1000, 9), (752, 480, 1000, 8, 1.0),
                 (752, 480, 1000, 8, 1.2, 0), (3000, 480, 1000)):
        with pytest.raises(sslib.SSError) as e:
            sslib.ss_orb_params_init(*args)
        assert e.value.status == sslib.SS_EINVAL
    assert "must" in sslib.ss_last_error()


def test_create_errors_without_valid_args(sslib):
    p = sslib.ss_orb_params_init(752, 480, 1000)
    with pytest.raises(sslib.SSError) as e:
        sslib.ss_create(0, p, 0)
    assert e.value.status == sslib.SS_EINVAL
    p.n_per_level[0] += 1  # tampered params are rejected
    with pytest.raises(sslib.SSError) as e:
        sslib.ss_create(0, p, 4)
    assert e.value.status == sslib.SS_EINVAL


def test_null_ctx_calls(sslib):
    with pytest.raises(sslib.SSError) as e:
        sslib.ss_orb_extract(None, 1, 0, 0, 752, 0, 0, 0)
    assert e.value.status == sslib.SS_EINVAL
    with pytest.raises(sslib.SSError):
        sslib.ss_destroy(None)


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_conext_dhakalrwcr22_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cpp", ".h", ".inc")):
                txt = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, fn
                assert "ss_oracle" not in txt and "brief_pattern_ref" not in txt, fn


def test_new_entry_points_reject_bad_args(sslib):
    """Round-2 entry points validate before touching the GPU."""
    L = sslib.lib()
    assert L.ss_track_run(None, 0, None, 1, None, None, 0, 1) == sslib.SS_EINVAL
    assert L.ss_brute_map_prepare(None, None, 10, None) == sslib.SS_EINVAL
    assert L.ss_orb_extract_frames(None, 1, None, None, None, None, None, None) == sslib.SS_EINVAL
    assert L.ss_debug_match_lanes(None, 3) == sslib.SS_EINVAL
    assert L.ss_debug_capture_samples(None, None) == sslib.SS_EINVAL
    assert L.ss_debug_distribution_paths(None, None, None) == sslib.SS_EINVAL
