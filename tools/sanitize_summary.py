"""Summarise a compute-sanitizer log: error kinds x (kernel, source line) with counts."""
import collections
import re
import sys

kinds = collections.Counter()
cur = None
for line in open(sys.argv[1], errors="replace"):
    m = re.match(r"========= (\S.*?)(?: of size \d+ bytes)?$", line.rstrip())
    if m and not line.startswith("=========     ") and "SUMMARY" not in line and "COMPUTE-SANITIZER" not in line:
        cur = [m.group(1), None, None]
        continue
    if cur is not None:
        a = re.match(r"=========     at (.*?) in (\S+:\d+)", line)
        if a and cur[1] is None:
            cur[1] = a.group(2)
        k = re.search(r"Device Frame: (?:void )?(hm::\S*?k_\w+(?:<[^>]*>)?)", line)
        if k and cur[2] is None:
            cur[2] = k.group(1)
        if line.startswith("=========     Saved host") or line.strip() == "=========":
            kinds[(cur[0], cur[1], cur[2])] += 1
            cur = None
for (kind, loc, kern), n in kinds.most_common():
    print(f"{n:8d}  {kind}  {loc}  {kern}")
