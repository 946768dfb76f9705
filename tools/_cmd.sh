python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/step_overhead.py 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > /tmp/b.json 2>/dev/null; python -c "
import json;d=json.load(open('/tmp/b.json')); print(d['value'], d['e2e']['value'], d['step_ms'], d['phases_ms'])"
