"""Per-step table of an INL_SSSP_TRACE file (the last source in it): kernel durations (us) from
the %globaltimer stamps, frontier sizes, relaxations and improvements per kernel and their rates."""
import sys

blocks, cur = [], None
for line in open(sys.argv[1]):
    if line.startswith("#"):
        cur = [line.strip(), []]
        blocks.append(cur)
    else:
        cur[1].append([int(x) for x in line.split()])
name, rows = blocks[-1]
print(name)
tot = [0.0] * 4
pr = pm = 0
for r in rows:
    i, t, nF, ns, rf, mf, rg, mg = r[0], r[1:7], r[7], r[8], r[9], r[10], r[11], r[12]
    pieces = r[13] if len(r) > 13 else 0
    if not t[0] or not t[4]:
        continue
    d = [(t[k + 1] - t[k]) / 1000 for k in range(4)]
    for k in range(4):
        tot[k] += d[k]
    ef, eg = rf - pr, rg - rf
    mfl, mgr = mf - pm, mg - mf
    pr, pm = rg, mg
    rate = lambda e, us: e / us / 1e3 if us > 0 else 0
    print(f"{i:3d} nF={nF:8d} ns={ns:8d} cmp={d[0]:6.1f} spl={d[1]:6.1f} flat={d[2]:7.1f} ({ef/1e6:7.2f}M e, {mfl/1e6:6.2f}M imp, {rate(ef, d[2]):5.1f} G/s)"
          f" grid={d[3]:7.1f} ({pieces:6d} pieces, {mgr/1e6:6.2f}M imp)")
print("totals us: compact %.0f split %.0f flat %.0f grid %.0f" % tuple(tot), "relaxed", pr, "improved", pm)
