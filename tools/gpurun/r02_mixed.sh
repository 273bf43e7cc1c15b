cd "$GRAFT_REPO_ROOT" || exit 1
run() { timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 5 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['staging'], d['value'], d['roofline']['frac'])"; }
echo "device(pull)"; run --staging device
echo "host"; run --staging host
for n in 1 2 3 4 6; do echo "mixed $n memop"; GSYS_COMPLETION=memop run --staging mixed --dev16 $n; done
for n in 2 4; do echo "mixed $n host-completion"; GSYS_COMPLETION=host run --staging mixed --dev16 $n; done
