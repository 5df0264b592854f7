"""Build libspp variants with compile-time knobs and time KC/KD on the GPU
(experiments only; the product build is paper_conf_ipps_ibrahimo22_b200/build.py).
usage: python scripts/variants.py build   (CPU)   |   python scripts/variants.py run (GPU)"""
import json
import os
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
VARIANTS = {
    "kc_alllanes": [],
    "kc_lane0": ["SPP_KC_ALL_LANES_RELEASE=0"],
}
# VARIANTS_JSON='{"name": ["DEFINE=1", ...], ...}' overrides the table (build and run)
if os.environ.get("VARIANTS_JSON"):
    VARIANTS = json.loads(os.environ["VARIANTS_JSON"])
OUT = ROOT / "paper_conf_ipps_ibrahimo22_b200" / "variants"


def build():
    import shutil
    from paper_conf_ipps_ibrahimo22_b200 import build as b
    shutil.rmtree(OUT, ignore_errors=True)        # only this sweep's libraries travel to the box
    for d in OUT.parent.glob("_build_*"):
        shutil.rmtree(d, ignore_errors=True)
    OUT.mkdir(exist_ok=True)
    for name, d in VARIANTS.items():
        b.build(force=True, defines=d, out=OUT / f"libspp_{name}.so")  # noqa
        print("built", name)


def run():
    res = {}
    names = [v for v in os.environ.get("VARIANT_NAMES", ",".join(VARIANTS)).split(",") if v]
    for name in names:
        env = dict(os.environ, SPP_LIB=str(OUT / f"libspp_{name}.so"))
        if "@" in name:
            env["SPP_L2_PERSIST_MB"] = name.split("@")[1]
        res[name] = {}
        if os.environ.get("VARIANT_COSMO", "1") == "1":
            out = subprocess.run([sys.executable, str(ROOT / "bench.py"), "--secondary", "none", "--cpu-seconds", "0.5",
                                  "--e2e-steps", "1", "--steps", "100",
                                  *os.environ.get("VARIANT_BENCH_ARGS", "").split()], env=env, capture_output=True,
                                 text=True)
            try:
                d = json.loads(out.stdout.strip().splitlines()[-1])
                res[name] = {"cosmo": d["value"], "frac": d["roofline"]["frac"]}
            except Exception as ex:
                res[name] = {"error": str(ex), "stderr": out.stderr[-500:]}
        if os.environ.get("VARIANT_DEEPCAM", "1") == "1":
            out = subprocess.run([sys.executable, str(ROOT / "bench.py"), "--workload", "deepcam", "--cpu-seconds",
                                  "0.5", "--e2e-steps", "1", "--steps", "10"], env=env, capture_output=True, text=True)
            try:
                d = json.loads(out.stdout.strip().splitlines()[-1])
                res[name].update({"deepcam": d["value"], "dfrac": d["roofline"]["frac"]})
            except Exception as ex:
                res[name]["derror"] = str(ex)
        if os.environ.get("VARIANT_SWEEP"):
            out = subprocess.run([sys.executable, str(ROOT / "scripts" / "sweep.py"), "--pool", "2", "--steps", "10",
                                  "--only", os.environ["VARIANT_SWEEP"]], env=env, capture_output=True, text=True)
            try:
                rows = json.loads(out.stdout)["rows"]
                res[name]["sweep"] = {f'{r["preset"]}/{r["policy"]}': round(r["frac_of_measured_hbm"], 3) for r in rows}
            except Exception as ex:
                res[name]["serror"] = str(ex) + out.stderr[-300:]
        print(name, res[name], flush=True)
    print(json.dumps(res))


if __name__ == "__main__":
    {"build": build, "run": run}[sys.argv[1]]()
