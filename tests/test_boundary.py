"""The C-ABI library loads and exports every function include/flep.h declares (no GPU needed),
and its host-only entry points behave (error codes, model evaluation)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_asplos_wulzj17_b200 import build, flep
    build.build()
    return flep.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "flep.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\*?\s+(flep_[a-z0-9_]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_boundary():
    names = declared_functions()
    for must in ("flep_init", "flep_register_kernel", "flep_launch", "flep_preempt", "flep_resume",
                 "flep_sync", "flep_query", "flep_shutdown", "flep_policy_arrive"):
        assert must in names
    assert len(names) >= 30


def test_library_exports_every_declared_symbol(lib):
    missing = [n for n in declared_functions() if not hasattr(lib, n)]
    assert missing == []


def test_binding_signatures_cover_the_header():
    from paper_conf_asplos_wulzj17_b200 import flep
    assert set(declared_functions()) == set(flep._SIG)


def test_host_only_entry_points(lib):
    from paper_conf_asplos_wulzj17_b200 import flep
    assert lib.flep_version().startswith(b"flep-b200")
    assert lib.flep_now_ns() > 0
    # NULL / invalid arguments return errors, never crash
    assert lib.flep_init(0, None, None) == flep.ERR_INVALID
    assert lib.flep_preempt(None, 1, 1) == flep.ERR_INVALID
    h = ctypes.c_void_p()
    assert lib.flep_policy_create(9, 148, ctypes.byref(h)) == flep.ERR_INVALID
    assert lib.flep_policy_create(2, 148, ctypes.byref(h)) == flep.OK
    assert lib.flep_policy_finish(h, 0, 77) == flep.ERR_INVALID    # unknown id
    assert lib.flep_policy_arrive(h, 0, 1, 0, 10, 0) == flep.OK
    assert lib.flep_policy_arrive(h, 1, 1, 0, 10, 0) == flep.ERR_INVALID    # duplicate id
    assert lib.flep_policy_destroy(h) == flep.OK
    assert b"duplicate" in lib.flep_last_error() or lib.flep_last_error() is not None


def test_model_predict_matches_oracle(lib):
    from oracle import estimates as E
    from paper_conf_asplos_wulzj17_b200 import flep
    for m in ([1.5, 0.25, 0.003, 2.0, 1000.0], [0, 0, 0, 0, 0.4], [-5, 0, 0, 0, 3], [1e-3, 2, 1e-4, 0, 12345.5]):
        for feat in ((8192, 256, 1 << 20, 0), (1, 1, 1, 1), (4096, 128, 10**8, 4096)):
            assert flep.model_predict_ns(m, *feat) == E.predict_ns(m, *feat)


def test_cuda_entry_points_fail_loudly_without_gpu(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_asplos_wulzj17_b200 import flep
    with pytest.raises(flep.FlepError) as e:
        flep.Runtime()
    assert e.value.status == flep.ERR_CUDA
