#!/bin/bash
# Walk CTAs per SM (SF_COPY_BPS): pack throughput vs requests landing during a walk
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/bps_build.log 2>&1 || { tail -20 gpurun_out/bps_build.log; exit 1; }
for b in 8 4 3 2 1; do
  SF_COPY_BPS=$b timeout 300 python scripts/pack_walk_ab.py 2>&1 | head -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())['probe']; print('bps', $b, {k: (round(v['pack_gbs']), round(v['unpack_gbs'])) for k, v in d.items() if isinstance(v, dict)})"
done
for b in 2 8 2 8; do SF_COPY_BPS=$b SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/bps_bench_$b.json 2>/dev/null
python - $b <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/bps_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]
print("bps", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms","preempt_to_resume_p50_ms")}, "e2e p99", round(d["e2e"]["value"],4),
      "pack GB/s", round(d["migration"]["pack_gbs"]), "nonpre wait/dev p50/p99", b["not_preempting"]["wait_p50"], b["not_preempting"]["wait_p99"], b["not_preempting"]["device_p50"], b["not_preempting"]["device_p99"],
      "pre dev p99", b["preempting"]["device_p99"])
PY
done
