"""SASS instructions per source line of one kernel (code-size / i-cache
work; run here on a -lineinfo cubin).

    python tools/sass_lines.py <nvdisasm -g output> <mangled kernel name> [N]
"""
import collections
import re
import sys


def main():
    path, kern = sys.argv[1], sys.argv[2]
    n = int(sys.argv[3]) if len(sys.argv) > 3 else 40
    fn = cur = None
    cnt = collections.defaultdict(collections.Counter)
    for l in open(path):
        m = re.match(r'\s*\.text\.(\S+):', l)
        if m:
            fn = m.group(1)
            continue
        m = re.search(r'## File "([^"]+)", line (\d+)', l)
        if m:
            cur = (m.group(1).split('/')[-1], int(m.group(2)))
            continue
        if re.match(r'\s+/\*[0-9a-f]{4,}\*/', l) and cur and fn:
            cnt[fn][cur] += 1
    c = cnt[kern]
    print("total", sum(c.values()))
    byf = collections.Counter()
    for (f, _), k in c.items():
        byf[f] += k
    print(byf.most_common())
    for (f, ln), k in c.most_common(n):
        print(k, f, ln)


if __name__ == "__main__":
    main()
