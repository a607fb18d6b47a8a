"""Summarise a scripts/km_trace timeline: per-tile period and median event offsets (cycles)
relative to the epilogue warp's loop top."""
import sys
import numpy as np
names = {0: 'conv after xfull', 1: 'conv after aempty', 2: 'conv after bempty', 3: 'conv done', 4: 'mma after afull',
         5: 'mma after dempty0', 6: 'mma after dempty1', 7: 'mma after ofull(i-1)', 8: 'mma done', 9: 'epi top',
         10: 'epi after xfull', 11: 'epi after dfull', 12: 'epi pass1 done', 13: 'mma issued h0', 14: 'mma issued h1',
         15: 'unused', 16: 'epi mask', 17: 'epi after fallback', 18: 'unused', 19: 'epi after oempty',
         20: 'epi end', 21: 'epiB top', 22: 'epiB after dfull', 23: 'epiB pass1 done', 24: 'unused',
         25: 'prod after xempty', 26: 'epi w7 end', 27: 'epi w8 end', 28: 'epi w9 end', 29: 'epi w7 pass1', 30: 'epi w8 pass1', 31: 'epi w9 pass1'}
rows = [list(map(int, l.split())) for l in open(sys.argv[1]) if not l.startswith('#')]
a = np.array(rows)[:, 1:]
# the two epilogue sets take alternate tiles: the set-B events (21-23) of odd tiles are folded onto
# the even rows (relative to the set-A loop top of the tile before)
if (a[0::2, 9] >= 0).all() and (a[1::2, 9] < 0).all():
    a = a.copy()
    ev = a[0::2]
    for e in (21, 22, 23):
        ev[:len(a[1::2]), e] = a[1::2, e]
    a = ev
top = a[:, 9]
print('period (per tile):', np.diff(top)[:24] / (2 if len(top) == 32 else 1))
med = {}
for ev in range(32):
    lo, hi = (5, 30) if len(top) == 32 else (10, 60)
    if (a[lo:hi, ev] >= 0).all():
        med[ev] = int(np.median(a[lo:hi, ev] - top[lo:hi]))
for ev, m in sorted(med.items(), key=lambda x: x[1]):
    print(f'   {names[ev]:24s} {m:7d}')
