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
    "kd_ns3": ["SPP_KD_WS_NS=3"],
    "kd_ns3_s2304": ["SPP_KD_WS_NS=3", "SPP_KD_WS_SLOT=2304"],
    "kd_ns4_s2304": ["SPP_KD_WS_NS=4", "SPP_KD_WS_SLOT=2304"],
    "kd_ns3_s3072": ["SPP_KD_WS_NS=3", "SPP_KD_WS_SLOT=3072"],
    "kd_ns3b": ["SPP_KD_WS_NS=3", "SPP_KD_TAG=1"],
}
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
                                  "--e2e-steps", "1", "--steps", "100"], env=env, capture_output=True, text=True)
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
        print(name, res[name], flush=True)
    print(json.dumps(res))


if __name__ == "__main__":
    {"build": build, "run": run}[sys.argv[1]]()
