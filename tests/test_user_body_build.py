"""The user-defined body extension (include/flep_body.cuh, flep_register_body) on the host: the
example body compiles for sm_100a against the public headers, its generated `<sym>_ops` fills the
table the runtime takes (ABI version, CTA size, argument size, all launchers), and libflep.so
exports flep_register_body. No GPU."""
import ctypes as C
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tests", "user_body", "body_affine_rev.cu")
OUT = os.path.join(ROOT, "tests", "user_body", "build", "libaffine_rev.so")


@pytest.fixture(scope="module")
def libs():
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    return F, build.build_user_body(SRC, OUT)


def test_user_body_compiles_and_fills_its_ops(libs):
    F, path = libs
    ul = C.CDLL(path)
    fill = ul.affine_rev_ops
    fill.restype = None
    fill.argtypes = [C.POINTER(F.BodyOps)]
    ops = F.BodyOps()
    fill(C.byref(ops))
    assert ops.abi_version == 1
    assert ops.threads == 128
    assert ops.args_size == 32                      # {int32_t* y; const int32_t* x; int32_t a, c; uint32_t n}
    assert ops.name == b"affine_rev"
    assert ops.clc and ops.sliced
    assert all(getattr(ops, f) for f in ("worker", "unwrapped", "static_launch", "occupancy", "clc", "sliced"))


def test_register_body_is_exported_and_checks_arguments(libs):
    F, _ = libs
    L = F.lib()
    assert hasattr(L, "flep_register_body")
    out = C.c_int32()
    assert L.flep_register_body(None, None, C.byref(out)) == F.ERR_INVALID
