#!/bin/bash
# e2e of the T40I10D10M pass for several raw-chunk periods of the packed upload (GPA_PACK_RAW_EVERY)
for r in ${@:-0 3 0 3 4}; do
  GPA_PACK_RAW_EVERY=$r GPA_TRACE=1 timeout 300 python bench.py --steps 10 --warmup 3 --no-ci --no-rules --no-cpu-baseline \
    > gpurun_out/pk_$r.json 2> gpurun_out/pk_$r.err
  python -c "import json; d=json.load(open('gpurun_out/pk_$r.json')); print('raw_every $r', 'e2e ms', round(d['e2e']['ms_per_step'], 2), 'dev ms', round(d['ms_per_step'], 2))"
  grep 'overlapped ingest' gpurun_out/pk_$r.err | tail -3 | sed 's/.*upload+hist+build+pairs/  upload+/; s/(pairs.*raw//'
done
