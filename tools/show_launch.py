"""Print the repo's kernels from an ncu --metrics gpu__time_duration.sum CSV launch list (us)."""
import csv
import sys

for path in sys.argv[1:]:
    print("==", path)
    h = None
    for r in csv.reader(open(path)):
        if "Kernel Name" in r:
            h = r
            continue
        if h and len(r) == len(h):
            d = dict(zip(h, r))
            if d.get("Metric Name") == "gpu__time_duration.sum" and "ifl::" in d["Kernel Name"]:
                name = d["Kernel Name"].split("(")[0].replace("void ", "").replace("ifl::<unnamed>::", "")
                print(f"  {name[:60]:60s} {float(d['Metric Value']) / 1e3:9.1f}")
