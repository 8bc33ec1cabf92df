"""CUDA-event timing helper shared by the study tools (not the product path)."""


def time_ms(fn, reps):
    """Median of `reps` CUDA-event timings of fn() on the current stream, after one warm-up call."""
    import torch
    fn()
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    out = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return out[len(out) // 2]
