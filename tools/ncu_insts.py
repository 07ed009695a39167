#!/usr/bin/env python3
"""Executed warp instructions per CUDA source line (and per SASS opcode) from
an ncu report with -lineinfo:  python tools/ncu_insts.py report.ncu-rep [N]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
fname, hdr = None, None
rows = []
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] in ('File Path', 'File Name'):
        fname = r[1].split('/')[-1]
        continue
    if r[0] == 'Line No':
        hdr = r
        continue
    if hdr and r[0].isdigit():
        try:
            n = int(r[hdr.index('Instructions Executed')] or 0)
        except ValueError:
            continue
        if n:
            rows.append((n, fname, int(r[0]), r[hdr.index('Source')].strip()[:90]))
tot = sum(x[0] for x in rows)
print("total warp instructions: %d" % tot)
for n, f, l, src in sorted(rows, reverse=True)[:top]:
    print("%5.1f%% %10d %s:%d  %s" % (100.0 * n / tot, n, f, l, src))
