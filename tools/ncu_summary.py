"""Summarise an ncu --set full report into JSON: python tools/ncu_summary.py rep.ncu-rep|raw.csv out.json"""
import csv, json, subprocess, sys
rep, out = sys.argv[1], sys.argv[2]
if rep.endswith(".csv"):  # already exported with `ncu -i rep --page raw --csv` (tools/ncu_export.sh)
    txt = open(rep).read()
else:
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(txt.splitlines()))
h, units, v = rows[0], rows[1], rows[2]
keep = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "launch__grid_size", "launch__block_size",
        "lts__t_requests_srcunit_tex_op_atom_dot_cas.sum", "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum",
        "smsp__cycles_active.avg", "sm__warps_active.avg.pct_of_peak_sustained_active"]
res = {k: (v[h.index(k)] + (" " + units[h.index(k)] if units[h.index(k)] else "")) for k in keep if k in h}
st = []
for i, n in enumerate(h):
    if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
        try:
            st.append((float(v[i]), n[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
        except ValueError:
            pass
tot = sum(x for x, _ in st) or 1.0
res["warp_stall_share_pct"] = {n: round(100 * x / tot, 1) for x, n in sorted(st, reverse=True)[:10]}
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res, indent=1))
