"""Per-opcode stall breakdown of one kernel from `ncu --page source --csv --print-source sass`."""
import csv, collections, sys

def load(path):
    rows = list(csv.reader(open(path)))
    h = rows[1]; ix = {n: i for i, n in enumerate(h)}
    data, seen = [], set()
    for r in rows[2:]:  # ncu may print the kernel's listing twice: keep one row per address
        if len(r) == len(h) and r[0] != 'Address' and r[0] not in seen:
            seen.add(r[0])
            data.append(r)
    return h, ix, data

def num(x):
    try: return float(x)
    except ValueError: return 0.0

def main(path, top=22):
    h, ix, data = load(path)
    stalls = [n for n in h if n.startswith('stall_') and 'Not Issued' not in n]
    tot = collections.Counter(); byop = collections.defaultdict(collections.Counter); samp = 0
    for r in data:
        samp += num(r[ix['Warp Stall Sampling (All Samples)']])
        t = r[ix['Source']].split(); op = t[0] if t else ''
        if op.startswith('@') and len(t) > 1: op = t[1]
        op = op.split('.')[0]
        for n in stalls:
            v = num(r[ix[n]]); tot[n] += v; byop[op][n] += v
        byop[op]['_n'] += 1; byop[op]['_exec'] += num(r[ix['Instructions Executed']])
    print('samples', samp)
    for n, v in tot.most_common(12): print(f'{n:28s} {v / samp * 100:6.2f}%')
    print()
    key = lambda kv: -sum(v for k, v in kv[1].items() if not k.startswith('_'))
    for op, c in sorted(byop.items(), key=key)[:top]:
        s = sum(v for k, v in c.items() if not k.startswith('_'))
        f = lambda k: c[k] / samp * 100
        print(f"{op:8s} n={c['_n']:5.0f} exec={c['_exec']:.2e} samp={s / samp * 100:5.1f}% wait={f('stall_wait'):5.1f} "
              f"sel={f('stall_selected'):5.1f} short={f('stall_short_sb'):5.1f} math={f('stall_math'):4.1f} "
              f"notsel={f('stall_not_selected'):4.1f} long={f('stall_long_sb'):4.1f} mio={f('stall_mio'):4.1f} disp={f('stall_dispatch'):4.1f}")

if __name__ == '__main__':
    main(sys.argv[1])
