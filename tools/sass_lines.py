"""SASS instruction count per source line for one kernel of a cubin (nvdisasm -g output): code-size audit."""
import re, sys
path, pat = sys.argv[1], sys.argv[2]
cur = None; cnt = {}; inside = False
for L in open(path):
    L = L.rstrip("\n")
    if L.strip().endswith(':') and 'kernel' in L and not L.strip().startswith('.L'):
        inside = pat in L
        continue
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', L)
    if m:
        cur = (m.group(1).split('/')[-1], int(m.group(2)))
        continue
    if re.match(r'\s+/\*[0-9a-f]+\*/', L) and cur:
        cnt[cur] = cnt.get(cur, 0) + 1
tot = sum(cnt.values())
print('total', tot)
for k, v in sorted(cnt.items(), key=lambda x: -x[1])[:int(sys.argv[3]) if len(sys.argv) > 3 else 25]:
    print(v, k)
