"""Summarise an ncu --set full raw CSV of GEMM kernels (cuBLAS beside the pair bodies): time,
achieved SM clock, tensor-pipe activity, L2 and fabric traffic, DRAM bytes. Usage:
python tools/ncu_gemm_summary.py raw.csv > summary.json"""
import csv
import json
import sys

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors_srcunit_tex_op_read.sum",
        "lts__t_requests_srcunit_tex_op_read.sum", "lts__t_requests_srcunit_tex_op_write.sum",
        "lts__t_requests_srcunit_ltcfabric.sum", "l1tex__m_xbar2l1tex_read_bytes.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__grid_size", "launch__cluster_size",
        "launch__shared_mem_per_block_dynamic", "launch__registers_per_thread"]


def main(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    head, units, data = rows[hi], rows[hi + 1], rows[hi + 2:]
    out = []
    for r in data:
        if len(r) != len(head):
            continue
        d = {"kernel": r[head.index("Kernel Name")][:90]}
        for k in KEYS:
            if k in head:
                i = head.index(k)
                d[k] = {"value": r[i], "unit": units[i]}
        out.append(d)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])
