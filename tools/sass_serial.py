"""Flags global loads that are issued one at a time: for each kernel of an
object file, the LDGs whose issue is preceded (since the previous LDG) by a
wait on the scoreboard that previous LDG writes -- the pattern a load inside
an if() produces in an unrolled gather.  usage: sass_serial.py file.o"""
import re
import subprocess
import sys


def main(obj):
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
    fn = None
    ins = []
    res = {}
    lines = sass.splitlines()
    for i, l in enumerate(lines):
        m = re.match(r"\s+Function : (\S+)", l)
        if m:
            fn = m.group(1)
            res[fn] = [0, 0]
            last_ldg_bar = None
            continue
        m = re.match(r"\s*/\*([0-9a-f]+)\*/\s+(.*?);\s*/\* (0x[0-9a-f]+) \*/", l)
        if not m or fn is None:
            continue
        m2 = re.search(r"/\* (0x[0-9a-f]+) \*/", lines[i + 1])
        ctrl = int(m2.group(1), 16) >> 41
        wbar, wmask = (ctrl >> 5) & 7, (ctrl >> 11) & 0x3F
        text = m.group(2)
        if last_ldg_bar is not None and wmask & (1 << last_ldg_bar):
            pending_wait = True
        else:
            pending_wait = False
        if "LDG" in text:
            res[fn][0] += 1
            if pending_wait_acc.get(fn):
                res[fn][1] += 1
            pending_wait_acc[fn] = False
            last_ldg_bar = wbar if wbar != 7 else None
        elif pending_wait:
            pending_wait_acc[fn] = True
    for fn, (n, s) in sorted(res.items(), key=lambda x: -x[1][1]):
        if n:
            print(f"{s:4d} / {n:4d} LDGs issued after a wait on the previous LDG  {fn[:110]}")


pending_wait_acc = {}
if __name__ == "__main__":
    main(sys.argv[1])
