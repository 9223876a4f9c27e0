"""Per-layer DRAM traffic of the R50 b32 set at HEAD from an ncu launch list
(run: ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum,lts__t_bytes_srcunit_tex_op_write.sum -k regex:k_tc_conv
--csv --log-file F python scripts/one_step_r50.py), written to
profiles/traffic_r50.json next to the algorithmic bytes.  usage:
traffic_r50.py NCU_CSV COMMIT"""
import csv
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets  # noqa: E402

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
idi = h.index("ID")
per = {}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1, "nsecond": 1e-3, "msecond": 1e3,
         "ns": 1e-3, "us": 1, "ms": 1e3, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}
for r in rows[1:]:
    try:
        val = float(r[vi].replace(",", ""))
    except ValueError:
        continue
    per.setdefault(int(r[idi]), {})[r[mi]] = val * scale.get(r[ui], 1)
launches = [per[k] for k in sorted(per)][-23:]  # the last step: one launch per layer
out = {"source": f"ncu launch list, commit {sys.argv[2]}, L2 flushed before each kernel (cold reads); "
                 "writes = bytes the kernel stores (TMA stores / L2 write sectors; dram__bytes_write misses lines still dirty in L2)",
       "layers": []}
tot_r = tot_w = tot_alg = 0.0
for L, m in zip(nets.RESNET50, launches):
    Ho, Wo = L.out_hw()
    alg_r = 2.0 * (32 * L.C * L.H * L.W + L.K * L.C * L.R * L.S)
    alg_w = 2.0 * 32 * L.K * Ho * Wo
    rd = m.get("dram__bytes_read.sum", 0.0)
    # bytes the kernel stores: TMA stores (the epilogue's main path), else L2 write sectors
    # (L2 write sectors count ~1.5-1.8x the TMA-stored bytes on B200 — the
    # L2 tag counter sees a write at more than one slice — so they are used
    # only for kernels without TMA stores, i.e. the generic writer)
    tma = m.get("l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum", 0.0)
    wr = tma if tma > 0 else 32.0 * m.get("lts__t_sectors_op_write.sum", 0.0)
    us = m.get("gpu__time_duration.sum", 0.0)
    us = us / 1e3 if us > 1e4 else us  # ncu reports ns or us
    out["layers"].append({"layer": L.name, "us": us, "dram_read": rd, "bytes_written": wr,
                          "alg_read": alg_r, "alg_write": alg_w})
    tot_r += rd
    tot_w += wr
    tot_alg += alg_r + alg_w
out["dram_bytes_per_step"] = tot_r + tot_w
out["dram_read_per_step"] = tot_r
out["write_per_step"] = tot_w
out["algorithmic_bytes_per_step"] = tot_alg
json.dump(out, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                 "traffic_r50.json"), "w"), indent=1)
print(json.dumps({k: v for k, v in out.items() if k != "layers"}))
