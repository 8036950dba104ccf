"""Measured-mode Identify (sg.measured_threshold) next to the model Identify on C2 / R-MAT 18 / C3 (f = 1 %):
the thresholds they pick and the measured Identify's wall time. python tools/measured_identify.py"""
import sys, time, json
sys.path.insert(0, '.')
import torch, sginputs as gen, paper_conf_icpp_hardhikbrks17_b200 as sg
for name, f in [(c, f) for c in ("C2", "R18", "C3") for f in (0.01, 0.1, 0.25)]:
    A = sg.DeviceCSR.from_host(gen.config(name))
    sg.measured_threshold(A, A, f, 99)  # warm
    torch.cuda.synchronize(); t0 = time.perf_counter()
    thr, rep = sg.measured_threshold(A, A, f, 1)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    thr_m = sg.sg_sample_threshold(A, A, f, 1)[0]
    print(json.dumps({"config": name, "f": f, "measured_thr": thr, "model_thr": thr_m, "identify_s": round(dt, 3),
                      "evaluations": len(rep["T_ms"]), "sample_rows": rep["sample_rows"]}), flush=True)
    del A; torch.cuda.empty_cache()
