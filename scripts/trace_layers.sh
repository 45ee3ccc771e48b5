cd "$(dirname "$0")/.."
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py -DQC_DEBUG > /dev/null 2>&1 || echo buildfail
for j in 16; do timeout 120 python scripts/trace_stem.py /tmp/tr.bin 4 $j 2>&1 | tail -14; done
