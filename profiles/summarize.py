"""Summarise ncu captures into committed text/JSON under profiles/ (gpurun_out/ is scratch).

    python profiles/summarize.py full  <report.ncu-rep>  <out_prefix>     # --set full capture -> metrics + stalls
    python profiles/summarize.py launches <launches.csv> <out_prefix>     # gpu__time_duration launch list -> shares
"""
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_atom.sum",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_red.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic"]


def full(rep, out):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    stalls = [h for h in hdr if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("_per_issue_active.ratio")]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k in KEYS:
            if k in hdr:
                d[k] = f"{r[hdr.index(k)]} {units[hdr.index(k)]}".strip()
        st = sorted(((float(r[hdr.index(h)] or 0), h) for h in stalls), reverse=True)[:6]
        d["top_stalls_per_issue"] = {h.replace("smsp__average_warps_issue_stalled_", "").replace(
            "_per_issue_active.ratio", ""): round(v, 2) for v, h in st}
        res.append(d)
    with open(out + ".json", "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


def launches(path, out):
    txt = open(path).read()
    txt = txt[txt.index('"ID"'):]
    rows = list(csv.DictReader(io.StringIO(txt)))
    agg = collections.defaultdict(list)
    for r in rows:
        agg[r["Kernel Name"].split("(")[0]].append(float(r["Metric Value"]) / 1e3)
    tot = sum(sum(v) for v in agg.values())
    lines = ["kernel | launches | mean us | total us | share", "---|---|---|---|---"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        lines.append(f"{k} | {len(v)} | {sum(v) / len(v):.2f} | {sum(v):.1f} | {100 * sum(v) / tot:.1f}%")
    s = "\n".join(lines)
    with open(out + ".md", "w") as f:
        f.write(f"ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised launches)\n"
                f"source: {path}\n\n" + s + "\n")
    print(s)


if __name__ == "__main__":
    {"full": full, "launches": launches}[sys.argv[1]](sys.argv[2], sys.argv[3])
