#!/bin/bash
# print bench summaries for files matching a prefix
for f in "$@"; do python3 -c "
import json,sys
try:
    d=json.load(open('$f'))
    print('$f'.split('/')[-1].ljust(28), 'step', round(d['ms_per_step'],4), 'sweep', round(d['roofline']['sweep_ms'],4), 'frac', round(d['roofline']['frac'],3), 'sort', round(d['stage_ms']['pack_sort_gather'],4), 'best', d['result']['best'])
except Exception as e: print('$f', 'ERR', e)
"; done
