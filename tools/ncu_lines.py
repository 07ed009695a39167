#!/usr/bin/env python3
"""Top source lines by warp-stall samples from an ncu report (needs -lineinfo):
   python tools/ncu_lines.py report.ncu-rep [N]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
fname = None
rows = []
hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == 'File Path':
        fname = r[1].split('/')[-1]
        continue
    if r[0] == 'Line No':
        hdr = r
        continue
    if hdr and r[0].isdigit():
        try:
            samples = int(r[hdr.index('Warp Stall Sampling (All Samples)')])
        except (ValueError, IndexError):
            continue
        stalls = {}
        for i, h in enumerate(hdr):
            if h.startswith('stall_') and '(' not in h:
                try:
                    v = int(r[i])
                except ValueError:
                    continue
                if v:
                    stalls[h[6:]] = v
        rows.append((samples, fname, int(r[0]), r[1].strip()[:70], stalls))
tot = sum(x[0] for x in rows) or 1
for s, f, ln, src, st in sorted(rows, reverse=True)[:top]:
    tops = ', '.join('%s %d' % kv for kv in sorted(st.items(), key=lambda kv: -kv[1])[:3])
    print('%5.1f%% %s:%d  %-70s  [%s]' % (100.0 * s / tot, f, ln, src, tops))
