"""Summarise an assign_sweep.sh log (debug lines + JSON lines)."""
import json
import re
import sys

dbg = None
rows = []
for l in open(sys.argv[1]).read().splitlines():
    if l.startswith('auction'):
        dbg = l
    if l.startswith('{'):
        r = json.loads(l)
        r['dbg'] = dbg
        rows.append(r)
for r in sorted(rows, key=lambda r: (r['cfg'], r['auction_s'])):
    e = r['env']
    m = re.search(r'steps=(\d+) phases=(\d+) gs_bids=(\d+) .*hist (.*)', r['dbg'])
    knobs = " ".join(f"{k.replace('PM_AUCTION_', '').lower()}={v}" for k, v in sorted(e.items()) if k != 'PM_AUCTION_DEBUG')
    print(r['cfg'], f"{r['auction_s']*1e3:7.1f} ms", knobs, "steps", m.group(1), "gs_bids", m.group(3), m.group(4))
