for fl in "" "-DACESO_EXPERIMENT_NO_PHASEB" "-DACESO_EXPERIMENT_NO_RC" "-DACESO_EXPERIMENT_NO_PHASEB -DACESO_EXPERIMENT_NO_RC"; do
  ACESO_NVCC_EXTRA="$fl" python -c "from paper_conf_eurosys_liumlsmybw24_b200 import buildlib; buildlib.build(force=True)" > /dev/null 2>&1
  r=$(python bench.py --no-cpu --no-e2e --no-dedup --no-incr --search-budget 0 --steps 400 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('%.3f Gcfg/s serial %.1f us' % (d['value']/1e9, d['roofline']['kernel_ms_serial']*1e3))")
  echo "[$fl] $r"
done
