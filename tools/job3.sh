mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
python tools/prof_one.py gpt3-1.3b 4096 3 --check 2>&1 | tail -4
ACESO_SCAN_NORESOLVE=1 python tools/prof_one.py gpt3-1.3b 4096 3 --check 2>&1 | tail -4
for v in "" "ACESO_SCAN_NORESOLVE=1" "ACESO_MINB=3" "ACESO_KERNEL=events"; do echo "== $v"; env $v python tools/prof_one.py gpt3-1.3b 65536 5 2>&1 | tail -2 | head -1; done
for w in gpt3-13b t5 wrn; do for v in "" "ACESO_KERNEL=events"; do echo "== $w $v"; env $v python tools/prof_one.py $w 65536 4 2>&1 | tail -2 | head -1; done; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 2 -c 1 -o gpurun_out/${TAG:-r2_scan} python tools/prof_one.py gpt3-1.3b 65536 3 > gpurun_out/ncu_scan.log 2>&1
tail -1 gpurun_out/ncu_scan.log
