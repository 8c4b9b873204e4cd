"""Per-kernel stall-reason totals and the hottest SASS lines from an ncu source page."""
import csv, subprocess, sys
def load(rep):
    if rep.endswith('.csv'):
        return list(csv.reader(open(rep).read().splitlines()))
    out = subprocess.run(['ncu','-i',rep,'--page','source','--csv','--print-source','sass'],capture_output=True,text=True).stdout
    return list(csv.reader(out.splitlines()))
def main(rep, top=40):
    rows = load(rep)
    hdr = rows[1]
    ia = hdr.index("Instructions Executed"); isrc = hdr.index("Source")
    scols = [i for i,h in enumerate(hdr) if h.startswith('stall_') and 'Not Issued' not in h]
    tot = {hdr[i]: 0 for i in scols}
    data = []
    ninst = 0
    for r in rows[2:]:
        if len(r) <= ia or not r[ia].isdigit(): continue
        ninst += int(r[ia])
        st = {hdr[i]: int(r[i]) if r[i].isdigit() else 0 for i in scols}
        for k, v in st.items(): tot[k] += v
        data.append((sum(st.values()), int(r[ia]), r[isrc].strip(), st))
    S = sum(tot.values())
    print('instructions executed', ninst, 'stall samples', S)
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        if v: print(f'  {k:28s} {100.0*v/S:6.2f}%')
    print('hottest lines (stall samples, executed, source, top reasons):')
    for s, n, src, st in sorted(data, key=lambda x: -x[0])[:top]:
        reasons = ','.join(f'{k[6:]}={v}' for k, v in sorted(st.items(), key=lambda x: -x[1])[:3] if v)
        print(f'  {s:7d} {n:11d}  {src[:60]:60s} {reasons}')
if __name__ == '__main__':
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)
