"""Summarise scripts/omb_window output (NEXT f2, reading C24): per (size, window) the
measured osu_bw rate and the error of the per-message model (C15) and of the window
model (C24) against it.  Usage: python scripts/omb_window_summary.py file.jsonl"""
import json
import sys

rows = [json.loads(x) for x in open(sys.argv[1])]
print(rows[0])
print(f"{'size':>8} {'w':>3} {'measured':>9} {'per-msg':>9} {'err':>7} {'window':>9} {'err':>7} same_cfg")
for r in rows[1:]:
    if "n" not in r or "bibw" in r:
        continue
    m = r["bw_window_cfg_GBps"]
    e1 = abs(r["pred_msg_GBps"] - m) / m * 100
    e2 = abs(r["pred_win_GBps"] - m) / m * 100
    print(f"{r['n'] >> 10:7d}K {r['w']:3d} {m:9.1f} {r['pred_msg_GBps']:9.1f} {e1:6.1f}% {r['pred_win_GBps']:9.1f} {e2:6.1f}% {r['same_cfg']}")
bib = [r for r in rows if r.get("bibw")]
if bib:
    print(f"{'size':>8} {'paths':>12} {'joint':>9} {'pred':>9} {'err':>7} {'indep':>9} {'pred':>9} {'err':>7}")
    for r in bib:
        e1 = abs(r["pred_joint_GBps"] - r["bibw_joint_GBps"]) / r["bibw_joint_GBps"] * 100
        e2 = abs(r["pred_independent_GBps"] - r["bibw_independent_GBps"]) / r["bibw_independent_GBps"] * 100
        print(f"{r['n'] >> 10:7d}K {r['mask']:>12} {r['bibw_joint_GBps']:9.1f} {r['pred_joint_GBps']:9.1f} {e1:6.1f}% "
              f"{r['bibw_independent_GBps']:9.1f} {r['pred_independent_GBps']:9.1f} {e2:6.1f}%")
for r in rows:
    if "select_miss_us" in r:
        print(r)
