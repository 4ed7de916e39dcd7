"""Extract one kernel's SASS from a cubin/.so (substring match on the function name)."""
import re
import subprocess
import sys

so, pat = sys.argv[1], sys.argv[2]
out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", so], capture_output=True, text=True).stdout
blocks = re.split(r"\n\s+Function : ", out)
for b in blocks[1:]:
    name = b.split("\n", 1)[0]
    if pat in name:
        print("Function :", b)
        break
