"""Print the SASS of one kernel of libsel.so (substring match on the mangled name)."""
import subprocess, sys
lib = sys.argv[2] if len(sys.argv) > 2 else "paper_conf_ipps_chikinaat19_b200/libsel.so"
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
blocks = out.split("\t\tFunction : ")
for b in blocks[1:]:
    name = b.split("\n", 1)[0]
    if sys.argv[1] in name:
        print(name)
        print(b)
        break
