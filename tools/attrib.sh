# Throughput attribution: bench with stages omitted (results invalid; timing only).
# Build the variants first (here, on CPU): tools/attrib.sh build
set -e
if [ "$1" = build ]; then
  mkdir -p build/variants
  for k in 1 2 3 4 7; do
    python - "$k" <<'PY'
import subprocess, sys
sys.path.insert(0, '.')
from paper_conf_ipps_rockenbachsgmtd19_b200 import build as b
k = sys.argv[1]
subprocess.check_call([b.NVCC, *b.FLAGS, f"-DDEDUP_ATTRIB_SKIP={k}", "-o",
                       f"build/variants/libdedup_skip{k}.so", *b.sources()])
PY
  done
  exit 0
fi
mkdir -p gpurun_out
set +e
for k in 0 1 2 3 4 7; do
  if [ $k = 0 ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_skip$k.so; fi
  DEDUP_LIB=$L timeout 300 python bench.py --steps 300 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/attrib_$k.log 2>&1
done
