import json, sys
for l in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweep.jsonl"):
    d = json.loads(l); r = d["roofline"]
    print(d["config"]["workload"][:34].ljust(34), d["config"].get("tile_rows"), "%8.4f ms" % r["kernel_ms"],
          "%7.1f GB/s" % r["achieved"], "frac %.3f" % r["frac"], "sm %s" % d["clocks"]["sm_mhz"])
