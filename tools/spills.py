"""Where does k_persistent spill?  (dev aid) python tools/spills.py [lib.so]"""
import os, re, subprocess, sys, tempfile
lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_icde_ahmady0gcz23_b200/lib/libkcore.so"
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
cub = [f for f in os.listdir(d) if f.startswith("kcore.") and f.endswith(".cubin")][0]
sass = subprocess.run(["nvdisasm", "-g", os.path.join(d, cub)], capture_output=True, text=True).stdout.split("\n")
secs = [i for i, l in enumerate(sass) if l.startswith("//---")]
for j, i in enumerate(secs):
    if ".text." in sass[i] and "k_persistent" in sass[i]:
        i1 = secs[j + 1] if j + 1 < len(secs) else len(sass)
        cur, cnt, tot = None, {}, 0
        for ll in sass[i:i1]:
            if ll.strip().startswith("//##") and "line" in ll:
                m = re.search(r'File "([^"]+)", line (\d+)', ll)
                if m:
                    cur = (os.path.basename(m.group(1)), int(m.group(2)))
            elif re.match(r"\s+/\*[0-9a-f]+\*/", ll):
                tot += 1
                if re.search(r"\b(STL|LDL)", ll):
                    k = (cur, "STL" if "STL" in ll else "LDL")
                    cnt[k] = cnt.get(k, 0) + 1
        print("instructions", tot)
        for k, v in sorted(cnt.items(), key=lambda x: -x[1])[:20]:
            print(v, k)
