"""Instruction mix (by SASS opcode) of one kernel in an ncu report, per unit of work.
usage: ncu_ops.py report.ncu-rep <substring of kernel name> [units] [top]"""
import collections
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
units = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
blocks, cur = [], None
for r in rows:
    if r and r[0] == 'Kernel Name':
        cur = [r[1], None, []]
        blocks.append(cur)
    elif cur is not None and cur[1] is None:
        cur[1] = r
    elif cur is not None:
        cur[2].append(r)
name, hdr, data = next(b for b in blocks if kern in b[0])
i_src, i_ex = hdr.index('Source'), hdr.index('Instructions Executed')
i_st = hdr.index('Warp Stall Sampling (All Samples)')
tot = sum(float(r[i_ex] or 0) for r in data)
ops, stall = collections.Counter(), collections.Counter()
for r in data:
    s = r[i_src].strip()
    if s.startswith('@'):
        s = s.split(None, 1)[1]
    op = s.split()[0] if s else '?'
    ops[op] += float(r[i_ex] or 0)
    stall[op] += float(r[i_st] or 0)
st_tot = sum(stall.values()) or 1
print(name[:90])
print(f'total {tot:.4g} instr, {tot / units:.2f} per unit')
for op, v in ops.most_common(top):
    print(f'{op:26s} {v / tot * 100:5.1f}%  {v / units:7.2f}/unit  stall {stall[op] / st_tot * 100:5.1f}%')
