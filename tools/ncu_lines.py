"""Warp instructions executed and stall samples per CUDA source line of one kernel in an ncu report
(needs -lineinfo). usage: ncu_lines.py report.ncu-rep [units] [top] [kernel substring]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
kern = sys.argv[4] if len(sys.argv) > 4 else None
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
fn, hdr, acc, keep = None, None, {}, True
src = {}
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == 'File Path':
        fn, hdr = r[1].split('/')[-1], None
        continue
    if r[0] == 'Function Name':
        keep = kern is None or kern in r[1]
        continue
    if r[0] == 'Line No':
        hdr = r
        continue
    if not keep or hdr is None or len(r) < len(hdr) or not r[0].strip().isdigit():
        continue
    try:
        n = float(r[hdr.index('Instructions Executed')] or 0)
        s = float(r[hdr.index('Warp Stall Sampling (All Samples)')] or 0)
    except ValueError:
        continue
    key = (fn, int(r[0]))
    a = acc.setdefault(key, [0.0, 0.0])
    a[0] += n
    a[1] += s
    src[key] = r[1].strip()[:80]
tot = sum(v[0] for v in acc.values())
stot = sum(v[1] for v in acc.values()) or 1
print(f"total {tot:.4g} warp-inst, {tot / units:.2f} per unit")
for k, v in sorted(acc.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{v[0] / units:7.3f}/unit {100 * v[1] / stot:5.1f}% stall  {k[0]}:{k[1]:<5d} {src[k]}")
