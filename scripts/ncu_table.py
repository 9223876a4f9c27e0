"""Per-launch table from an ncu report holding many launches (raw page), for
profiles/.  Usage: python scripts/ncu_table.py REPORT.ncu-rep OUT.txt [TRAFFIC.json]

TRAFFIC.json gets {"dram_bytes_per_step": sum over the launches of
dram__bytes_read.sum + dram__bytes_write.sum, "launches": n, "source": report}
(the bench's roofline.traffic)."""
import csv
import json
import subprocess
import sys

COLS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "launch__grid_size", "launch__registers_per_thread"]


def to_num(v, unit):
    try:
        x = float(v.replace(",", ""))
    except Exception:
        return None
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
             "nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "ns": 1e-3, "us": 1.0, "ms": 1e3}
    return x * scale.get(unit, 1.0)


def main():
    rep, out = sys.argv[1], sys.argv[2]
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    h, units = rows[0], rows[1]
    ki = h.index("Kernel Name")
    lines, tot_t, tot_b = [], 0.0, 0.0
    lines.append(f"# {rep}\n# idx  kernel  time_us  dram_MB  tensor%  sm%  L2_MB  grid  regs")
    for n, r in enumerate(rows[2:]):
        vals = {}
        for c in COLS:
            if c in h:
                i = h.index(c)
                vals[c] = to_num(r[i], units[i])
        t = vals.get("gpu__time_duration.sum") or 0.0
        b = (vals.get("dram__bytes_read.sum") or 0.0) + (vals.get("dram__bytes_write.sum") or 0.0)
        tot_t += t
        tot_b += b
        lines.append(f"{n:3d}  {r[ki][:48]:48s} {t:9.2f} {b / 1e6:9.2f} "
                     f"{vals.get(COLS[3]) or 0:6.1f} {vals.get(COLS[4]) or 0:6.1f} "
                     f"{(vals.get('lts__t_bytes.sum') or 0) / 1e6:9.1f} {vals.get('launch__grid_size') or 0:6.0f} "
                     f"{vals.get('launch__registers_per_thread') or 0:4.0f}")
    lines.append(f"# total: {len(rows) - 2} launches, {tot_t:.1f} us (serialised, cold), "
                 f"{tot_b / 1e6:.1f} MB DRAM")
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))
    if len(sys.argv) > 3:
        with open(sys.argv[3], "w") as f:
            json.dump({"dram_bytes_per_step": tot_b, "launches": len(rows) - 2, "source": rep,
                       "serialised_us": tot_t}, f, indent=1)


if __name__ == "__main__":
    main()
