"""The C-ABI library loads and exports every symbol include/sq.h declares (no GPU needed)."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "sq.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sq_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for required in ["sq_quantize_groups", "sq_pack", "sq_linear_prefill", "sq_linear_decode",
                     "sq_stage_forward", "sq_pipeline_run"]:
        assert required in names


def test_library_exports_every_declared_symbol():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    lib = ctypes.CDLL(sq.LIB_PATH)
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing


def test_host_only_functions():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    L = sq.lib()
    assert L.sq_abi_version() == 3
    # (4 h1^2 + 2 h1 h2) * bit/8 bytes per layer
    h1 = 9216
    for bits in (3, 4, 8, 16):
        tot = (L.sq_packed_bytes(3 * h1, h1, bits) + L.sq_packed_bytes(h1, h1, bits)
               + L.sq_packed_bytes(4 * h1, h1, bits) + L.sq_packed_bytes(h1, 4 * h1, bits))
        assert tot == (4 * h1 * h1 + 2 * h1 * 4 * h1) * bits // 8
    assert L.sq_packed_bytes(8, 128, 5) == 0
    assert L.sq_meta_bytes(8, 256, 128) == 8 * 2 * 4


def test_invalid_arguments_rejected_before_launch():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    L = sq.lib()
    st = L.sq_quantize_groups(None, 8, 128, 5, 128, None, None, None, None)
    assert st == sq.SQ_EINVAL and b"bits" in L.sq_last_error()
    w = sq.sq_qweight(4, 64, 16, 128, 16, 16, None)
    st = L.sq_linear_decode(ctypes.byref(w), None, 128, 1, None, 8, 0, None, None, 0, None)
    assert st == sq.SQ_ENOTSUP
    w = sq.sq_qweight(4, 128, 16, 100, 16, 16, None)
    st = L.sq_linear_decode(ctypes.byref(w), None, 128, 1, None, 8, 0, None, None, 0, None)
    assert st == sq.SQ_EINVAL


def test_indicator_arguments_rejected_before_launch():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    L = sq.lib()
    bits = (ctypes.c_int32 * 2)(4, 9)
    st = L.sq_scale_sq_sums(None, 8, 128, 128, bits, 2, None, None, 0, None)
    assert st == sq.SQ_EINVAL and b"bits" in L.sq_last_error()
    st = L.sq_scale_sq_sums(None, 8, 100, 128, bits, 1, None, None, 0, None)
    assert st == sq.SQ_EINVAL
    assert L.sq_scale_sq_sums_workspace_bytes(8, 100) == 0
    assert L.sq_act_moments(None, 0, None, None, 0, None) == sq.SQ_EINVAL
