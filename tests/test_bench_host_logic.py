"""Host logic of the bench configs (no GPU): the co-run case list of the paper's Figs. 8, 10-12
(E4 / E6 / E8) and the queue kernels' registration options."""
import bench_configs as BC


class _F:                                            # the body ids register options depend on
    BODY_GEMM_BF16, BODY_GEMM_BF16_2SM, BODY_GEMM_BF16_2SM_W = 6, 9, 10
    BODY_SPMV_CSR_F32, BODY_STENCIL5_F32, BODY_SAXPY_F32 = 3, 4, 2


def test_corun_cases_cover_the_paper_experiments():
    cases = BC.corun_cases()
    by = {}
    for exp, name, trace in cases:
        by.setdefault(exp, []).append((name, trace))
    assert {e: len(v) for e, v in by.items()} == {"E4": 16, "E6": 16, "E8": 28}
    # E4: every large LP kernel with every small HP kernel, the HP arriving after the LP
    for name, tr in by["E4"]:
        assert [j["size_class"] for j in tr] == [2, 1]
        assert [j["priority"] for j in tr] == [0, 1]
        assert tr[0]["arrival_ns"] < tr[1]["arrival_ns"]
    assert len({n for n, _ in by["E4"]}) == 16
    # E6: the same pairs at equal priority
    assert {n for n, _ in by["E6"]} == {n for n, _ in by["E4"]}
    assert all(j["priority"] == 0 for _, tr in by["E6"] for j in tr)
    # E8: A large then B, C small (B != C), distinct triplets, the paper's VA_SPMV_MM among them
    names = [n for n, _ in by["E8"]]
    assert len(set(names)) == 28 and "VA_SPMV_MM" in names
    for name, tr in by["E8"]:
        assert [j["size_class"] for j in tr] == [2, 1, 1]
        assert tr[1]["type"] != tr[2]["type"]
        assert tr[0]["arrival_ns"] < tr[1]["arrival_ns"] < tr[2]["arrival_ns"]
    assert BC.corun_cases() == cases                  # seeded


def test_queue_kernel_options(monkeypatch):
    monkeypatch.delenv("FLEP_QUEUE_FETCH", raising=False)
    o = BC._qopts(_F, "spmv", _F.BODY_SPMV_CSR_F32)
    assert o["spec_fetch"] and not o["prefetch"] and o["chunk"] == 2 and not o["in_tile"]
    o = BC._qopts(_F, "gemm_bf16", _F.BODY_GEMM_BF16)
    assert o["in_tile"] and not o["spec_fetch"]
    assert BC._qopts(_F, "gemm_bf16", _F.BODY_GEMM_BF16_2SM_W)["in_tile"]
    o = BC._qopts(_F, "saxpy_f32", _F.BODY_SAXPY_F32)
    assert o["chunk"] == 8 and not o["spec_fetch"]
    monkeypatch.setenv("FLEP_QUEUE_FETCH", "prefetch")
    o = BC._qopts(_F, "stencil_f32", _F.BODY_STENCIL5_F32)
    assert o["prefetch"] and not o["spec_fetch"]
