# GPU call: pipeline depth (slots) under the driver's 20-step command, interleaved reps.
mkdir -p gpurun_out
rm -f gpurun_out/slots.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2 3; do for n in 16 24 32 40; do
  echo "slots $n $(timeout 300 python bench.py --steps ${STEPS:-20} --warmup 5 --step-only --slots $n 2>&1 | grep -o '"value": [0-9.]*')" >> gpurun_out/slots.log
done; done
echo done
