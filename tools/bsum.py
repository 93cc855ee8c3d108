import json,sys
for f in sys.argv[1:]:
    try:
        d=json.load(open(f))
        r=d["roofline"]
        print(f.split('/')[-1], round(d["value"]/1e9,3),"G/s", round(d["ms_per_step"],2),"ms frac",round(r["frac"],3),"sgd_ms",round(r["sgd_ms_per_epoch"],2),"rmse",round(d["test_rmse"],5),"clk",d["clocks"]["sm_mhz"])
    except Exception as e: print(f, "ERR", e)
