#!/bin/bash
# Write profiles/<TAG>_ncu_summary.md from gpurun_out/*_<TAG>* (the outputs of tools/profile_round.sh TAG).
# Usage: tools/write_summary.sh TAG "title suffix"
TAG=$1; TITLE=${2:-}
cd "$(dirname "$0")/.."
{
echo "# Round 1 ncu evidence, refresh $TAG $TITLE"
echo
echo "Captured with \`tools/profile_round.sh $TAG\` (ncu --set full --clock-control none --import-source on, one launch after warm-up; launch lists with \`--metrics gpu__time_duration.sum --clock-control none\`). Per-launch, cold-cache, serialised: compare shares, not absolute times."
echo
echo "Bench lines of the same build (no profiler, same box, \`gpurun_out/bench_*_$TAG.json\`):"
echo
echo "| config | compress GB/s | ratio | chunk_kernel ms | roofline frac (alu) | decompress GB/s | e2e GB/s | version 2 GB/s | CPU oracle GB/s (threads) | SM MHz / throttle |"
echo "|---|---|---|---|---|---|---|---|---|---|"
for f in bench_full_$TAG bench_c3_$TAG bench_c4_$TAG bench_c5_$TAG; do python -c "
import json; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1])
v=d.get('versions',{}).get('2',{}).get('value')
c=d.get('cpu_baseline')
cs='%.3f (%d)' % (c['value'], c['cores']) if c else '-'
print('| %s | %.1f | %.4f | %.3f | %.3f | %.1f | %.1f | %s | %s | %s %s |' % (d['config']['workload'].split(':')[0], d['value'], d['ratio'], d['kernels_ms']['chunk'], d['roofline']['frac'], d['decompress']['value'], d['e2e']['value'], '%.2f'%v if v else '-', cs, d['clocks']['sm_mhz'], d['clocks']['reasons'] or 'none'))"; done
python -c "
import json; d=json.loads(open('gpurun_out/bench_full_$TAG.json').read().strip().splitlines()[-1]); c=d['cpu_baseline']
print(); print('CPU oracle beside it (c2, same run): %.3f GB/s on %d threads (%s).' % (c['value'], c['cores'], c['sample']))
r=json.loads(open('gpurun_out/bench_ref_$TAG.json').read().strip().splitlines()[-1]); print('Reference arm (\`--impl reference\`, the oracle): %.3f GB/s on %d threads.' % (r['value'], r['cpu_baseline']['cores']))
n=json.loads(open('gpurun_out/bench_n2gloo_$TAG.json').read().strip().splitlines()[-1]); print('N=2 code path (gloo, two ranks sharing the one GPU): %.1f GB/s aggregate, sharded decompression %.1f GB/s, round trip exact: %s.' % (n['value'], n['decompress']['value'], n['decompress']['roundtrip_exact']))"
echo
echo "## Launch list, compress only (bench.py default config c2_csource_128m, --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-decompress --no-versions; torch L2-flush fill kernels included)"
echo
python tools/ncu_summary.py launches gpurun_out/launches_$TAG.csv
echo
echo "## Launch list with the decompress leg"
echo
python tools/ncu_summary.py launches gpurun_out/launches_dec_$TAG.csv
echo
echo "## Fused chunk kernel (rows a1-a4), --set full"
for cfg in c2_csource_128m c4_random_1g c3_runs20_1g; do echo; python tools/ncu_summary.py full gpurun_out/full_${cfg}_$TAG.ncu-rep $cfg; done
echo
echo "### Per-phase split of the c2 chunk kernel (tools/ncu_lines.py: warp instructions / warp stall samples by source line range)"
echo
echo '```'
python tools/ncu_lines.py gpurun_out/full_c2_csource_128m_$TAG.ncu-rep lzss_chunk.cu ${RANGES:-56:138:helpers 139:244:walk 245:306:v2 307:376:stage 377:473:build 474:515:mask 516:569:fixup 570:648:emit 649:736:scan+write} --top 15
echo '```'
echo
echo "## Decoder (row a6), --set full, c2 stream"
for k in walk_kernel decode_kernel; do echo; python tools/ncu_summary.py full gpurun_out/full_${k}_c2_$TAG.ncu-rep $k; done
} > profiles/${TAG}_ncu_summary.md 2>&1
cp gpurun_out/launches_$TAG.csv profiles/${TAG}_launches.csv
cp gpurun_out/launches_dec_$TAG.csv profiles/${TAG}_launches_dec.csv
