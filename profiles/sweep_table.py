"""Table of the SURVEY §8(d) sensitivity sweep (profiles/sweep_run.sh bench lines) -> markdown on stdout."""
import glob
import json
import os
import sys

d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweep"
pts = {}
for f in glob.glob(os.path.join(d, "*.json")):
    try:
        j = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    c = j["config"]
    v = "fused" if "fused" in c["variant"] else "two-pass"
    pts[(c["n_att"], c["n_instr"], v)] = j
print("| n_att | n_instr | fused s/iter (k_fused3 frac) | two-pass s/iter (aprod1 / aprod2 frac) | SM MHz (fused / two-pass) |")
print("|---|---|---|---|---|")
for na in sorted({k[0] for k in pts}):
    for ni in sorted({k[1] for k in pts if k[0] == na}):
        f, t = pts.get((na, ni, "fused")), pts.get((na, ni, "two-pass"))
        fs = f"{f['value']:.3e} ({f['roofline']['frac']:.2f})" if f else "—"
        ts = (f"{t['value']:.3e} ({t['iteration_roofline']['aprod1_frac']:.2f} / "
              f"{t['iteration_roofline']['aprod2_frac']:.2f})") if t else "—"
        ck = f"{int(f['clocks']['sm_mhz']) if f else '—'} / {int(t['clocks']['sm_mhz']) if t else '—'}"
        print(f"| {na:,} | {ni:,} | {fs} | {ts} | {ck} |")
